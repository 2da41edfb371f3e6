"""GPU check of the partitioned grid tail (part.cu): parity vs the oracle on a few graphs in the
part modes, then C3 step times with and without it (GP_DEBUG traces of the tail levels)."""
import os
import sys
import time
import traceback

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import torch  # noqa: E402

import graphgen as G  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_goodarzibg16_b200.gp as gp  # noqa: E402
from gpu_helpers import assert_levels_equal, gpu_coarsen  # noqa: E402

MODES = {
    "part": {"GP_SMALL": "0"},
    "part_many": {"GP_SMALL": "0", "GP_PART_W": "256"},
    "part_global": {"GP_SMALL": "0", "GP_PART_W": "256", "GP_PART_GARCS": "1", "GP_PART_WCAP": "64"},
    "part_gstage": {"GP_SMALL": "0", "GP_PART_GSTAGE": "1"},
}
KN = ("GP_SMALL", "GP_PART_W", "GP_PART_GARCS", "GP_PART_WCAP", "GP_PART", "GP_PART_GSTAGE")


def star(k, wmax=100):
    e = [(0, i, 1 + (i * 37) % wmax) for i in range(1, k + 1)] + [(i, i + 1, 1 + (i * 11) % wmax) for i in range(1, k)]
    return G.from_edge_list(k + 1, e)


cases = {
    "grid40": (lambda: G.grid2d(40, 40), 10),
    "C1": (lambda: G.make_config("C1"), 100),
    "delaunay128": (lambda: G.delaunay_like(128), 100),
    "rmat10": (lambda: G.varied_vwgt(G.shuffle_rows(G.rmat(10), 3)), 10),
    "star5000": (lambda: star(5000), 2),
    "delaunay512": (lambda: G.delaunay_like(512), 100),
    "rgg2^16": (lambda: G.rgg(1 << 16), 100),
}
only = sys.argv[1:] if len(sys.argv) > 1 else None
ctx = gp.Context(0)
for name, (mk, thr) in cases.items():
    if only and name not in only:
        continue
    g = mk()
    ref = oracle.coarsen_to(g, threshold=thr)
    for mode, env in MODES.items():
        for k in KN:
            os.environ.pop(k, None)
        os.environ.update(env)
        try:
            got = gpu_coarsen(gp, ctx, g, threshold=thr)
            assert_levels_equal(got, ref, f"{name} {mode}")
            print(f"OK   {name} {mode}: {len(ref)} levels", flush=True)
        except Exception as ex:  # noqa: BLE001
            print(f"FAIL {name} {mode}: {str(ex)[:300]}", flush=True)
            if "CUDA" in str(ex) or "cuda" in str(ex):
                traceback.print_exc()
                sys.exit(1)
for k in KN:
    os.environ.pop(k, None)
# timing: C3 with / without the grid tail
g = G.make_config("C3", device="cuda")
graph = gp.Graph.create(ctx, g["adjp"], g["adjncy"], g["adjwgt"], g["vwgt"])
for setting in ("0", "1", "0", "1"):
    os.environ["GP_PART"] = setting
    ts = []
    for rep in range(8):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        h = graph.coarsen_to(100)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        nl = len(h)
        h.close()
    print(f"C3 GP_PART={setting}: {sorted(ts)[len(ts)//2]:.3f} ms median, {nl} levels", flush=True)
