"""Small loopback (simulated multi-rank) coarsening vs the oracle; for compute-sanitizer runs.

usage: python scripts/debug_dist.py [G] [graph]   graph in grid8 | del32 | rmat10
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np  # noqa: E402

import graphgen as G  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_goodarzibg16_b200.gp as gp  # noqa: E402
from gpu_helpers import gpu_coarsen  # noqa: E402

nr = int(sys.argv[1]) if len(sys.argv) > 1 else 2
name = sys.argv[2] if len(sys.argv) > 2 else "grid8"
g = {"grid8": lambda: G.grid2d(8, 8, unit=True), "del32": lambda: G.delaunay_like(32),
     "rmat10": lambda: G.rmat(10, 8)}[name]()
ctx = gp.Context(0, loopback=nr)
ref = oracle.coarsen_to(g, threshold=4)
got = gpu_coarsen(gp, ctx, g, threshold=4)
print("levels", len(got), len(ref))
for i, (a, b) in enumerate(zip(got, ref)):
    ok = {k: bool(np.array_equal(a[k], b[k])) for k in ("match", "cmap")}
    okc = {k: bool(np.array_equal(a["coarse"][k], b["coarse"][k])) for k in ("adjp", "adjncy", "adjwgt", "vwgt")}
    print(i, a["n"], b["n"], a["rounds"], b["rounds"], ok, okc)
