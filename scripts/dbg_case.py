"""Reproduce one random-graph case (n m seed wmax) through gp_coarsen_to, compare with the oracle."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import graphgen as G  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_goodarzibg16_b200.gp as gp  # noqa: E402
from gpu_helpers import assert_levels_equal, gpu_coarsen  # noqa: E402

n, m, seed, wmax = (int(x) for x in sys.argv[1:5])
thr = int(sys.argv[5]) if len(sys.argv) > 5 else 100
g = G.random_graph(n, m, seed, wmax)
ctx = gp.Context(0)
ref = oracle.coarsen_to(g, thr)
got = gpu_coarsen(gp, ctx, g, thr)
assert_levels_equal(got, ref, "case")
print("OK", len(ref), "levels")
