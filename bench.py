#!/usr/bin/env python
"""Benchmark of the GP-metis coarsening hot path on B200 (one JSON line on rank 0).

A "step" is one full coarsen-to-threshold (gp_coarsen_to: every level's matching rounds,
cmap, contraction and CSR assembly) of the BASELINE.json workload, input resident in HBM.

  metric  fine edges coarsened/s = sum over levels of |E_level| / (time of one step)
  value   whole-job aggregate over all ranks
  e2e     the same metric through the C ABI with HOST buffers: pinned H2D of the CSR,
          gp_graph_create + gp_coarsen_to, D2H of every level's cmap + the coarsest graph
  roofline  dominant kernel family, algorithmic bytes / CUDA-event time
  levels    per level: n, nnz, rounds, match / contract us, edges/s, §8(d) bytes, GB/s, fraction
  level0    the level-0 match / contract roofline fractions (north_star's target)
  cpu_baseline  the oracle (oracle/, single thread) on the box's host, bounded sample

--impl reference times the oracle (the reference arm of this tier) on the same config.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import graphgen as G  # noqa: E402

WORKLOADS = {
    "C1": ("grid64x64_unit", 100),
    "C2": ("rgg_n2^20_deg13_w1-100", 100),
    "C3": ("delaunay_like_n2^22_w1-100", 100),
    "C4": ("rmat_s24_ef16_w1-4", 100),
    "C5": ("road_like_n2^26_deg2.5_w1-10", 100),
}
METRIC = "fine edges coarsened/sec (sum of |E| over levels / full coarsen-to-threshold time)"
UNIT = "edges/s"
L2_BYTES = 126 * 1024 * 1024


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


# ------------------------------------------------------------------------------------------
# algorithmic byte model per kernel family: SURVEY.md §8(d), int32 everywhere
# ------------------------------------------------------------------------------------------
def level_bytes(l) -> dict:
    """Compulsory HBM bytes of one level, from the device counters the level
    reports: S = arcs scanned by the proposals (all rounds, round 1 included), V_s = rows
    scanned, L = live vertex visits of the commits, R = rounds.

      A1 degree binning        12 n
      A2 propose               8 S + 12 V_s + min(4 (S - nnz), 4 n (R - 1))
      A3 commit                12 L
      A5 cmap                  12 n + 4 n_c
      A6-A8 contraction        12 n + 8 nnz + 4 n + 8 cnnz + 12 n_c   (single-pass assembly)

    match = A1 + A2 + A3 (k_match_level), contract = A5 + A6-A8 (k_contract_level).
    """
    n, nnz, nc, cnnz = l["n"], l["nnz"], l["n_coarse"], l["cnnz"]
    S, Vs, R, L = l["arcs_scanned"], l["rows_scanned"], max(l["rounds"], 1), l["live_visits"]
    a1 = 12 * n
    a2 = 8 * S + 12 * Vs + min(4 * max(S - nnz, 0), 4 * n * (R - 1))
    a3 = 12 * L
    a5 = 12 * n + 4 * nc
    a678 = 12 * n + 8 * nnz + 4 * n + 8 * cnnz + 12 * nc
    return {"match": a1 + a2 + a3, "contract": a5 + a678}


def ncu_traffic(config: str, kernel: str):
    """DRAM bytes (read + write) per step of `kernel` from the committed ncu launch list
    (profiles/r1/ncu_traffic_<config>.json, written by scripts/summarize_profiles.py from one
    profiled gp_coarsen_to), or None when no capture of this config is committed."""
    for rnd in ("r2", "r1"):
        path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles", rnd, f"ncu_traffic_{config}.json")
        try:
            j = json.load(open(path))
            return float(j["kernels"][kernel]["dram_bytes"]), f"profiles/{rnd}/" + os.path.basename(path)
        except Exception:
            continue
    return None


# ------------------------------------------------------------------------------------------
# clocks sampled during the timed region
# ------------------------------------------------------------------------------------------
class ClockSampler:
    FIELDS = "clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown," \
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap"

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "20"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
            # the timed region starts only once the sampler is producing samples (nvidia-smi
            # takes ~0.1-0.5 s to start; a short region would otherwise see none)
            t0 = time.time()
            while not self.lines and time.time() - t0 < 5.0:
                time.sleep(0.01)
            self.skip = len(self.lines)  # samples taken before the region are not counted
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], 0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines[getattr(self, "skip", 0):]:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 6:
                continue
            try:
                sm.append(float(parts[0]))
                mx = max(mx, float(parts[1]))
            except ValueError:
                continue
            for nm, val in zip(names, parts[2:6]):
                if val.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------------------------------
# oracle timing (cpu_baseline and --impl reference)
# ------------------------------------------------------------------------------------------
def oracle_run(g, threshold, tie_seed=0, max_rounds=0):
    import oracle
    t0 = time.perf_counter()
    levels = oracle.coarsen_to(g, threshold, tie_seed=tie_seed, max_rounds=max_rounds)
    dt = time.perf_counter() - t0
    return dt, sum(l["nnz"] // 2 for l in levels), len(levels)


def cpu_baseline(g, threshold, budget_s=12.0, tie_seed=0, max_rounds=0):
    runs, tot_t, tot_e, nlev = 0, 0.0, 0, 0
    while runs == 0 or tot_t < budget_s:
        dt, e, nlev = oracle_run(g, threshold, tie_seed, max_rounds)
        runs += 1
        tot_t += dt
        tot_e += e
        if runs >= 8:
            break
    return {"value": tot_e / tot_t, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"{runs} full coarsen-to-{threshold} run(s) of the same graph ({nlev} levels), "
                      f"single-threaded C oracle, {tot_t:.1f} s"}


def host_info():
    try:
        model = [l.split(":", 1)[1].strip() for l in open("/proc/cpuinfo") if l.startswith("model name")][0]
    except Exception:
        model = "unknown"
    return {"host_cpu": model, "host_nproc": os.cpu_count()}


# ------------------------------------------------------------------------------------------
def make_graph(cfg: str, device: str):
    t0 = time.perf_counter()
    g = G.make_config(cfg, device=device)
    return g, time.perf_counter() - t0


def run_ours(args, rank, world, local_rank):
    import paper_conf_ipps_goodarzibg16_b200.gp as gp
    torch.cuda.set_device(local_rank)
    dev = f"cuda:{local_rank}"
    name, threshold = WORKLOADS[args.config]
    g, gen_s = make_graph(args.config, dev)
    n, nnz = g["n"], g["nnz"]
    sharded = world > 1   # N GPUs: the sharded path over NCCL (strong scaling: one graph)
    if sharded:
        uid = [gp.nccl_unique_id() if rank == 0 else None]
        torch.distributed.broadcast_object_list(uid, src=0)
        ctx = gp.Context(local_rank, nccl_id=uid[0], rank=rank, nranks=world)
        vb, ve = n * rank // world, n * (rank + 1) // world   # this rank's vertex range
        a0, a1 = int(g["adjp"][vb]), int(g["adjp"][ve])
        shard = {"adjp": (g["adjp"][vb:ve + 1] - a0).contiguous(), "adjncy": g["adjncy"][a0:a1].contiguous(),
                 "adjwgt": g["adjwgt"][a0:a1].contiguous(), "vwgt": g["vwgt"][vb:ve].contiguous()}
        graph = gp.Graph.create_dist(ctx, n, vb, shard["adjp"], shard["adjncy"], shard["adjwgt"], shard["vwgt"])
    elif args.loopback > 1:  # the sharded protocol simulated on this one GPU (tests / profiling)
        ctx = gp.Context(local_rank, loopback=args.loopback)
        graph = gp.Graph.create(ctx, g["adjp"], g["adjncy"], g["adjwgt"], g["vwgt"])
    else:
        ctx = gp.Context(local_rank)
        graph = gp.Graph.create(ctx, g["adjp"], g["adjncy"], g["adjwgt"], g["vwgt"])
    stream = ctx.stream

    def step():
        return graph.coarsen_to(threshold, tie_seed=args.tie_seed, max_rounds=args.max_rounds)

    # warm-up
    hier = None
    for _ in range(args.warmup):
        hier = step()
        levels = [vars(l) for l in hier.levels()]
        hier.close()
    levels = [{k: v for k, v in l.items() if k != "coarse"} for l in levels]
    edges_per_step = sum(l["nnz"] // 2 for l in levels)

    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    ctx.reset_stats()
    ctx.set_timing(True)
    launches0 = ctx.launch_count()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    with ClockSampler(local_rank) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            hier = step()
            hier.close()
        ev1.record(stream)
        torch.cuda.synchronize()
    ms = ev0.elapsed_time(ev1)
    launches = ctx.launch_count() - launches0
    kstats = ctx.kernel_stats()
    ltimes = ctx.launch_times()   # (kind, ms) of every launch of the timed steps, in order
    ctx.set_timing(False)
    # untimed-instrumentation check: the same steps without event brackets
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        hier = step()
        hier.close()
    e1.record(stream)
    torch.cuda.synchronize()
    ms_plain = e0.elapsed_time(e1)
    ms_step = min(ms, ms_plain) / args.steps
    if world > 1:
        t = torch.tensor([ms_step], device=dev)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        ms_step = float(t.item())

    # per-level rows (BASELINE metric "fine edges coarsened/sec per level"): each step enqueues
    # level l's matching then its contraction (speculative levels after the stop come last);
    # the median over the timed steps of each launch's CUDA-event time
    peak, peak_kind = peaks()
    per_step = len(ltimes) // args.steps if args.steps else 0
    level_rows, tail = [], None
    nreg, nreg_known = len(levels), False
    if not sharded and args.loopback <= 1 and per_step >= 1:
        # levels on the level kernels: 2 launches each (propose = k_match_level, contract =
        # k_contract_level); the coarse-level tail (one 'other' launch) runs the rest
        step0 = ltimes[:per_step]
        nreg, nreg_known = 0, True
        while 2 * nreg + 1 < per_step and nreg < len(levels) and step0[2 * nreg][0] == "propose" \
                and step0[2 * nreg + 1][0] == "contract":
            nreg += 1
        for i in range(nreg):
            l = levels[i]
            t = {}
            for fam, off in (("match", 0), ("contract", 1)):
                t[fam] = statistics.median(ltimes[st * per_step + 2 * i + off][1] for st in range(args.steps))
            b = level_bytes(l)
            tl = t["match"] + t["contract"]
            level_rows.append({
                "level": i, "n": l["n"], "nnz": l["nnz"], "n_coarse": l["n_coarse"], "cnnz": l["cnnz"],
                "rounds": l["rounds"], "match_us": round(1e3 * t["match"], 2), "contract_us": round(1e3 * t["contract"], 2),
                "edges_per_s": (l["nnz"] // 2) / (tl / 1e3),
                "bytes_match": b["match"], "bytes_contract": b["contract"],
                "GBps_match": b["match"] / (t["match"] / 1e3) / 1e9, "GBps_contract": b["contract"] / (t["contract"] / 1e3) / 1e9,
                "frac_match": b["match"] / (t["match"] / 1e3) / 1e9 / peak,
                "frac_contract": b["contract"] / (t["contract"] / 1e3) / 1e9 / peak})
        if nreg < len(levels) and 2 * nreg < per_step and step0[2 * nreg][0] == "other":
            tus = 1e3 * statistics.median(ltimes[st * per_step + 2 * nreg][1] for st in range(args.steps))
            rest = levels[nreg:]
            tb = sum(sum(level_bytes(l).values()) for l in rest)  # §8(d) bytes of the tail's levels
            tail = {"levels": [nreg, len(levels) - 1], "launches": 1, "us": round(tus, 2),
                    "n_first": rest[0]["n"], "edges": sum(l["nnz"] // 2 for l in rest),
                    "rounds": [l["rounds"] for l in rest],
                    "edges_per_s": sum(l["nnz"] // 2 for l in rest) / (tus / 1e6),
                    "bytes": tb, "GBps": tb / (tus / 1e6) / 1e9,
                    "kernel": ("coarse-level tail: k_part (every SM, each CTA's vertex range and rows in shared "
                               "memory) when the level fits the SMs' shared memory, k_small (one CTA) when it fits one "
                               "SM, k_medium (one cluster, opt-in)")}

    # roofline of the dominant kernel family
    # (the levels the two level kernels ran; the coarse-level tail's levels are one other launch)
    fam_bytes = {}
    for l in (levels[:nreg] if nreg_known else levels):
        for k, v in level_bytes(l).items():
            fam_bytes[k] = fam_bytes.get(k, 0) + v
    if sharded:  # global sizes / world: the bytes one rank's kernels move (rows split evenly)
        fam_bytes = {k: v / world for k, v in fam_bytes.items()}
    kfam = {"match": "propose", "contract": "contract"}   # gp_kernel_kind of each family
    fam_ms = {k: kstats[kfam[k]]["ms"] / args.steps for k in fam_bytes}
    if tail is not None:  # the coarse-level tail is one launch: its own family
        fam_bytes["tail"] = tail["bytes"]
        fam_ms["tail"] = tail["us"] / 1e3
    dom = max(fam_ms, key=lambda k: fam_ms[k])
    achieved = fam_bytes[dom] / (fam_ms[dom] / 1e3) / 1e9 if fam_ms[dom] > 0 else 0.0
    step_bytes = sum(fam_bytes.values())
    traffic = ncu_traffic(args.config, {"match": "k_match_level", "contract": "k_contract_level",
                                        "tail": "k_part"}[dom])

    # projection: a synthetic labelling of the coarsest graph (c mod 64)
    # carried down to level 0 in one launch; algorithmic bytes = CM_0 read + labels written +
    # every coarser CM and the coarse labels read once
    proj = None
    if not sharded and args.loopback <= 1:
        hp = step()
        nl = len(hp)
        pc = (torch.arange(levels[-1]["n_coarse"], device=dev, dtype=torch.int32) % 64).contiguous()
        pf = torch.empty(n, dtype=torch.int32, device=dev)
        for _ in range(3):
            hp.project(pc, pf)
        reps = 20
        torch.cuda.synchronize()
        p0 = torch.cuda.Event(enable_timing=True)
        p1 = torch.cuda.Event(enable_timing=True)
        p0.record(stream)
        for _ in range(reps):
            hp.project(pc, pf)
        p1.record(stream)
        torch.cuda.synchronize()
        pms = p0.elapsed_time(p1) / reps
        pbytes = 8 * n + sum(4 * l["n"] for l in levels[1:]) + 4 * levels[-1]["n_coarse"]
        proj = {"levels": nl, "ms": pms, "bytes": pbytes, "GB/s": pbytes / (pms / 1e3) / 1e9,
                "frac": pbytes / (pms / 1e3) / 1e9 / peaks()[0], "launches": 1,
                "l2": "CM_0 + labels 2x16.8 MiB; coarser CMs L2-resident after the first rep"}
        # un-coarsening: project + refine level by level from the same
        # synthetic coarsest labelling, k = 64, 3 % imbalance (P22.s35); CUDA events, best of 3
        part0 = torch.empty(n, dtype=torch.int32, device=dev)
        um = []
        moves = 0
        for _ in range(3):
            torch.cuda.synchronize()
            u0 = torch.cuda.Event(enable_timing=True)
            u1 = torch.cuda.Event(enable_timing=True)
            u0.record(stream)
            moves = hp.uncoarsen(graph, pc, part0, 64, imbalance_pct=3, max_passes=8)
            u1.record(stream)
            torch.cuda.synchronize()
            um.append(u0.elapsed_time(u1))
        src = torch.repeat_interleave(torch.arange(n, device=dev), torch.diff(g["adjp"].long()))
        cut_ref = int(g["adjwgt"][part0[src] != part0[g["adjncy"].long()]].sum().item()) // 2
        cut_proj = int(g["adjwgt"][pf[src] != pf[g["adjncy"].long()]].sum().item()) // 2
        proj["uncoarsen"] = {"nparts": 64, "imbalance_pct": 3, "ms": min(um), "moves": moves,
                             "edge_cut_projected": cut_proj, "edge_cut_refined": cut_ref,
                             "start": "coarsest graph labelled c mod 64 (synthetic; initial partitioning is out of scope)"}
        del src
        hp.close()

    # end-to-end through the C ABI with host buffers
    host = {k: (shard if sharded else g)[k].cpu().pin_memory() for k in ("adjp", "adjncy", "adjwgt", "vwgt")}
    h2d = sum(t.numel() * 4 for t in host.values())
    # pinned result buffers sized from the warm-up hierarchy (what a partitioner keeps:
    # every level's CM for projection, and the coarsest graph)
    cm_bufs = [torch.empty(l["n_local"] if sharded else l["n"], dtype=torch.int32).pin_memory() for l in levels]
    e2e_ms = []
    d2h = 0
    for it in range(max(2, min(args.steps, 5)) + 1):
        torch.cuda.synchronize()
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        if sharded:
            gh = gp.Graph.create_dist(ctx, n, vb, host["adjp"], host["adjncy"], host["adjwgt"], host["vwgt"])
        else:
            gh = gp.Graph.create(ctx, host["adjp"], host["adjncy"], host["adjwgt"], host["vwgt"])
        hh = gh.coarsen_to(threshold, tie_seed=args.tie_seed, max_rounds=args.max_rounds)
        nb = 0
        for i in range(len(hh)):
            _, c = hh.download_level(i, cmap=cm_bufs[i], want_match=False)
            nb += c.numel() * 4
        last = hh.download_coarse(len(hh) - 1)
        nb += sum(last[k].numel() * 4 for k in ("adjp", "adjncy", "adjwgt", "vwgt"))
        b.record(stream)
        torch.cuda.synchronize()
        hh.close()
        gh.close()
        if it > 0:
            e2e_ms.append(a.elapsed_time(b))
        d2h = nb
    e2e_step = min(e2e_ms)

    line = {
        "metric": METRIC, "value": edges_per_step / (ms_step / 1e3), "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
        "scaling": "strong" if sharded else "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
        "config": {"workload": f"{args.config}:{name}" + (f":rm_seed{args.tie_seed:#x}" if args.tie_seed else "")
                   + (f":max_rounds{args.max_rounds}" if args.max_rounds else ""), "n": n, "edges": nnz // 2, "threshold": threshold,
                   "levels": len(levels), "edges_all_levels": edges_per_step,
                   "level0_edges_per_s": level_rows[0]["edges_per_s"] if level_rows else None,
                   "t_full_ms": ms_step, "rounds": [l["rounds"] for l in levels],
                   "n_final": levels[-1]["n_coarse"], "stop_reason": levels[-1]["stop_reason"],
                   "shrink_per_level": [round(l["n_coarse"] / l["n"], 4) for l in levels],
                   "l2": f"L0 input {(4 * (2 * nnz + 2 * n)) / 2**20:.0f} MiB > L2 126 MiB (no flush)",
                   "parallelism": (f"sharded x{world}: vertex ranges, NCCL all-gather per handshake round"
                                   if sharded else f"loopback x{args.loopback} on 1 GPU (sharded protocol simulated)"
                                   if args.loopback > 1 else "single GPU"),
                   "gen_s": round(gen_s, 2)},
        "hbm_gbs_step": step_bytes / (ms_step / 1e3) / 1e9,
        # north_star's target: >= 50 % of HBM roofline on the matching and contraction kernels of
        # the 2^22 mesh -- their level-0 launches, SURVEY §8(d) bytes / CUDA-event time
        "level0": ({"match_frac": level_rows[0]["frac_match"], "contract_frac": level_rows[0]["frac_contract"],
                    "match_us": level_rows[0]["match_us"], "contract_us": level_rows[0]["contract_us"],
                    "edges_per_s": level_rows[0]["edges_per_s"], "peak_GBps": peak, "peak_kind": peak_kind}
                   if level_rows else None),
        "levels": level_rows,
        "tail": tail,
        "roofline": {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak, "peak_kind": peak_kind,
                     "unit": "GB/s", "frac": achieved / peak,
                     "traffic": traffic[0] if traffic else None,
                     "traffic_source": traffic[1] if traffic else None,
                     "bytes_per_step": fam_bytes[dom], "ms_per_step": fam_ms[dom]},
        "kernels": {k: {"ms_per_step": fam_ms[k], "GB/s": (fam_bytes[k] / (fam_ms[k] / 1e3) / 1e9) if fam_ms[k] else None,
                        "launches_per_step": (kstats[kfam[k]]["launches"] / args.steps) if k in kfam else 1.0}
                    for k in fam_bytes},
        "e2e": {"value": edges_per_step / (e2e_step / 1e3), "unit": UNIT, "ms_per_step": e2e_step,
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h},
        "gpu_launches": launches,
        "projection": proj,
        "clocks": clk.summary(),
    }
    if rank == 0 and not args.no_cpu_baseline:
        gh = {k: g[k].cpu() for k in ("adjp", "adjncy", "adjwgt", "vwgt")}
        line["cpu_baseline"] = cpu_baseline(gh, threshold, tie_seed=args.tie_seed, max_rounds=args.max_rounds)
        line["cpu_baseline"].update(host_info())
    graph.close()
    ctx.close()
    return line


def run_reference(args, rank, world):
    name, threshold = WORKLOADS[args.config]
    if rank != 0:
        return None
    g, _ = make_graph(args.config, "cpu")
    for _ in range(args.warmup):
        oracle_run(g, threshold, args.tie_seed, args.max_rounds)
    t = 0.0
    e = 0
    for _ in range(args.steps):
        dt, e, nlev = oracle_run(g, threshold, args.tie_seed, args.max_rounds)
        t += dt
    ms = t / args.steps * 1e3
    value = e / (ms / 1e3)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": f"{args.config}:{name}" + (f":rm_seed{args.tie_seed:#x}" if args.tie_seed else "")
                       + (f":max_rounds{args.max_rounds}" if args.max_rounds else ""), "n": g["n"], "edges": g["nnz"] // 2,
                       "threshold": threshold, "edges_all_levels": e},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"full coarsen-to-{threshold} per step, single-threaded C oracle"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    line["cpu_baseline"].update(host_info())
    return line


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", choices=sorted(WORKLOADS), default="C3")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--max-rounds", type=int, default=0,
                    help="cap the handshake rounds per level (1 = the paper's one-shot HEM + conflict pass, P18.s7-13)")
    ap.add_argument("--loopback", type=int, default=0,
                    help="run the sharded protocol with this many simulated ranks on one GPU")
    ap.add_argument("--tie-seed", type=lambda x: int(x, 0), default=0,
                    help="0: lower id wins equal-weight ties (north_star); else the RM tie priority "
                         "lowbias32(v ^ seed) (DESIGN R17, P18.s8)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3) if args.impl == "ours" else args.warmup

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1 and args.impl == "ours":
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        torch.distributed.init_process_group("nccl", device_id=torch.device(f"cuda:{local_rank}"))

    if args.impl == "reference":
        line = run_reference(args, rank, world)
    else:
        line = run_ours(args, rank, world, local_rank)
    if rank == 0 and line is not None:
        print(json.dumps(line), flush=True)
    if world > 1 and args.impl == "ours":
        torch.distributed.barrier()
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
