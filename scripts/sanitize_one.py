"""One small coarsen_to under compute-sanitizer (debugging aid)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as G  # noqa: E402
import paper_conf_ipps_goodarzibg16_b200.gp as gp  # noqa: E402

ctx = gp.Context(0)
g = G.delaunay_like(int(sys.argv[1]) if len(sys.argv) > 1 else 64)
d = {k: g[k].cuda() for k in ("adjp", "adjncy", "adjwgt", "vwgt")}
Gr = gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"])
h = Gr.coarsen_to(100)
print("levels", len(h))
