"""One warm-up + one profiled gp_coarsen_to of a config (for ncu launch lists / captures).

usage: python scripts/profile_once.py [C3] [--reps N]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import graphgen as G  # noqa: E402
import paper_conf_ipps_goodarzibg16_b200.gp as gp  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
reps = int(sys.argv[sys.argv.index("--reps") + 1]) if "--reps" in sys.argv else 1
g = G.make_config(cfg, device="cuda")
ctx = gp.Context(0)
graph = gp.Graph.create(ctx, g["adjp"], g["adjncy"], g["adjwgt"], g["vwgt"])
torch.cuda.synchronize()
h = graph.coarsen_to(100)   # warm-up
print("warm-up launches", ctx.launch_count(), flush=True)
h.close()
torch.cuda.cudart().cudaProfilerStart()
for _ in range(reps):
    h = graph.coarsen_to(100)
    h.close()
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
print("total launches", ctx.launch_count())
