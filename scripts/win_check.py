"""GPU check of the windowed big-level matching (match_win.cu): parity vs the oracle with the
window path forced on small graphs (GP_WIN_N), then C3/C2/C5 step times with / without it."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import torch  # noqa: E402

import graphgen as G  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_goodarzibg16_b200.gp as gp  # noqa: E402
from gpu_helpers import assert_levels_equal, gpu_coarsen  # noqa: E402

ctx = gp.Context(0)
if "--parity" in sys.argv:
    os.environ["GP_WIN_N"] = "2000"
    cases = {
        "delaunay128": (lambda: G.delaunay_like(128), 100, {}),
        "delaunay512": (lambda: G.delaunay_like(512), 100, {}),
        "delaunay512_rm": (lambda: G.delaunay_like(512), 100, {"tie_seed": 0x9E3779B9}),
        "delaunay512_cap2": (lambda: G.delaunay_like(512), 100, {"max_rounds": 2}),
        "rgg2^16": (lambda: G.rgg(1 << 16), 100, {}),
        "road256": (lambda: G.road_like(256), 100, {}),
        "grid_shuf_vw": (lambda: G.varied_vwgt(G.shuffle_rows(G.grid2d(200, 200), 5)), 50, {}),
    }
    for name, (mk, thr, kw) in cases.items():
        g = mk()
        ref = oracle.coarsen_to(g, threshold=thr, **kw)
        for part in ("1", "0"):
            os.environ["GP_PART"] = part
            try:
                got = gpu_coarsen(gp, ctx, g, threshold=thr, **kw)
                assert_levels_equal(got, ref, f"{name} part={part}")
                print(f"OK   {name} part={part}: {len(ref)} levels", flush=True)
            except Exception as ex:  # noqa: BLE001
                print(f"FAIL {name} part={part}: {str(ex)[:300]}", flush=True)
    os.environ.pop("GP_WIN_N")
    os.environ.pop("GP_PART", None)
for cfg in [c for c in ("C3", "C2", "C5") if c in sys.argv]:
    g = G.make_config(cfg, device="cuda")
    graph = gp.Graph.create(ctx, g["adjp"], g["adjncy"], g["adjwgt"], g["vwgt"])
    for setting in ("0", "1", "0", "1"):
        os.environ["GP_WIN"] = setting
        ts = []
        for rep in range(10):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            h = graph.coarsen_to(100)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
            nl = len(h)
            h.close()
        print(f"{cfg} GP_WIN={setting}: {sorted(ts)[len(ts)//2]:.3f} ms median, {nl} levels", flush=True)
    graph.close()
