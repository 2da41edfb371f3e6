"""Small coarsen_to runs for compute-sanitizer (memcheck / racecheck / synccheck), each checked
bit for bit against the oracle so that a sanitizer run also proves the results:
    python scripts/sanitize_cases.py c3_256 | star5000 | loopback3"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import graphgen as G  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_goodarzibg16_b200.gp as gp  # noqa: E402
from gpu_helpers import assert_levels_equal, gpu_coarsen  # noqa: E402

case = sys.argv[1]
if case == "c3_256":
    ctx, g, thr = gp.Context(0), G.delaunay_like(256), 100
elif case == "star5000":
    edges = [(0, i, 1 + (i * 37) % 100) for i in range(1, 5001)] + [(i, i + 1, 1 + (i * 11) % 100) for i in range(1, 5000)]
    ctx, g, thr = gp.Context(0), G.from_edge_list(5001, edges), 2
elif case == "loopback3":
    ctx, g, thr = gp.Context(0, loopback=3), G.delaunay_like(64), 20
else:
    raise SystemExit(f"unknown case {case}")
got = gpu_coarsen(gp, ctx, g, threshold=thr)
assert_levels_equal(got, oracle.coarsen_to(g, threshold=thr), case)
print(f"{case}: {len(got)} levels bit-exact vs the oracle")
