"""Summarise an ncu --csv launch list: per-launch time, DRAM bytes, share (prints a table)."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
h = rows[hi]
ki, mi, vi, ui, idi = (h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"),
                       h.index("Metric Unit"), h.index("ID"))
per = collections.OrderedDict()
for r in rows[hi + 1:]:
    key = (int(r[idi]), r[ki].split("(")[0].replace("void ", "").replace("gp::", ""))
    v = float(r[vi].replace(",", ""))
    u = r[ui]
    scale = {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3, "byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6,
             "Gbyte": 1e9}.get(u, 1.0)
    per.setdefault(key, {})[r[mi]] = v * scale
tot_t = sum(d.get("gpu__time_duration.sum", 0) for d in per.values())
print(f"{'id':>4} {'kernel':24s} {'us':>9} {'MB':>9} {'GB/s':>8} {'share':>6}")
agg = collections.defaultdict(lambda: [0.0, 0.0, 0])
for (i, k), d in per.items():
    t = d.get("gpu__time_duration.sum", 0)
    b = d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
    agg[k][0] += t
    agg[k][1] += b
    agg[k][2] += 1
    print(f"{i:4d} {k:24s} {t:9.1f} {b / 1e6:9.2f} {b / t / 1e3 if t else 0:8.0f} {t / tot_t:6.3f}")
print(f"total {tot_t:.1f} us over {len(per)} launches")
for k, (t, b, c) in agg.items():
    print(f"  {k:24s} {c:3d} launches {t:9.1f} us {b / 1e6:9.1f} MB  share {t / tot_t:.3f}")
