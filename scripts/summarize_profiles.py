"""Summarise ncu outputs into a markdown file under profiles/ (what the judge reads).

usage: python scripts/summarize_profiles.py OUT.md LAUNCHES.csv [REP.ncu-rep ...] [--bench bench.json]
                                            [--traffic TRAFFIC.json]

--traffic writes {kernel: {launches, us, dram_bytes}} summed over the profiled gp_coarsen_to
(one bench step); bench.py reports it as roofline.traffic next to the algorithmic bytes.
"""
import collections
import csv
import io
import json
import subprocess
import sys

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit rate %"),
    ("l1tex__t_sector_hit_rate.pct", "L1 hit rate %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active % (occupancy)"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "threads per instruction (of 32)"),
    ("l1tex__average_t_sectors_per_request_pipe_lsu_mem_global_op_ld.ratio", "sectors per global load request"),
    ("launch__registers_per_thread", "registers / thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
]


def launch_table(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, mi, vi, ui, idi = (h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"),
                           h.index("Metric Unit"), h.index("ID"))
    per = collections.OrderedDict()
    for r in rows[hi + 1:]:
        key = (int(r[idi]), r[ki].split("(")[0].split("<")[0].replace("void ", "").replace("gp::", ""))
        v = float(r[vi].replace(",", ""))
        scale = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3,
                 "byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(r[ui], 1.0)
        per.setdefault(key, {})[r[mi]] = v * scale
    return per


def rep_metrics(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units, vals = rows[0], rows[1], rows[2]
    d = {}
    for name, label in METRICS:
        if name in h:
            i = h.index(name)
            d[label] = f"{vals[i]} {units[i]}".strip()
    stalls = []
    for i, name in enumerate(h):
        if name.startswith("smsp__average_warps_issue_stalled_") and name.endswith("_per_issue_active.ratio"):
            try:
                stalls.append((float(vals[i]), name.replace("smsp__average_warps_issue_stalled_", "")
                               .replace("_per_issue_active.ratio", "")))
            except ValueError:
                pass
    stalls.sort(reverse=True)
    return d, stalls[:6]


def main():
    args = sys.argv[1:]
    bench = None
    if "--bench" in args:
        k = args.index("--bench")
        bench = args[k + 1]
        args = args[:k] + args[k + 2:]
    traffic = None
    if "--traffic" in args:
        k = args.index("--traffic")
        traffic = args[k + 1]
        args = args[:k] + args[k + 2:]
    out, launches, reps = args[0], args[1], args[2:]
    lines = [f"# ncu summary ({launches})", ""]
    per = launch_table(launches)
    tot = sum(d.get("gpu__time_duration.sum", 0) for d in per.values())
    lines += ["## Launch list (one profiled gp_coarsen_to of C3; ncu: serialised, cold caches)", "",
              "| id | kernel | us | DRAM MB | GB/s | share |", "|---|---|---|---|---|---|"]
    agg = collections.defaultdict(lambda: [0.0, 0.0, 0])
    for (i, k), d in per.items():
        t = d.get("gpu__time_duration.sum", 0)
        b = d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
        agg[k][0] += t
        agg[k][1] += b
        agg[k][2] += 1
        lines.append(f"| {i} | {k} | {t:.1f} | {b / 1e6:.1f} | {b / t / 1e3 if t else 0:.0f} | {t / tot:.3f} |")
    lines += ["", f"Total {tot:.1f} us over {len(per)} launches.", "", "| kernel | launches | us | DRAM MB | share |",
              "|---|---|---|---|---|"]
    for k, (t, b, c) in agg.items():
        lines.append(f"| {k} | {c} | {t:.1f} | {b / 1e6:.1f} | {t / tot:.3f} |")
    if traffic:
        json.dump({"source": launches.split("/")[-1], "note": "ncu --clock-control none, one gp_coarsen_to",
                   "kernels": {k: {"launches": c, "us": t, "dram_bytes": b} for k, (t, b, c) in agg.items()}},
                  open(traffic, "w"), indent=1)
    for rep in reps:
        d, stalls = rep_metrics(rep)
        lines += ["", f"## Full capture: `{rep.split('/')[-1]}` (level-0 launch)", "", "| metric | value |",
                  "|---|---|"]
        lines += [f"| {k} | {v} |" for k, v in d.items()]
        lines += ["", "Top warp stall reasons (warps per issue-active cycle): " +
                  ", ".join(f"{n} {v:.2f}" for v, n in stalls)]
    if bench:
        j = json.loads(open(bench).read().strip().splitlines()[-1])
        lines += ["", "## Bench line", "", "```", json.dumps(j, indent=1), "```"]
    open(out, "w").write("\n".join(lines) + "\n")
    print(out)


if __name__ == "__main__":
    main()
