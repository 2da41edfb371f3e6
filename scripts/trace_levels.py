"""Per-level, per-phase device timestamps of gp_coarsen_to (GP_DEBUG=1 must be set)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as G  # noqa: E402
import paper_conf_ipps_goodarzibg16_b200.gp as gp  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
g = G.make_config(cfg, device="cuda")
ctx = gp.Context(0)
graph = gp.Graph.create(ctx, g["adjp"], g["adjncy"], g["adjwgt"], g["vwgt"])
for rep in range(3):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    h = graph.coarsen_to(100)
    e1.record()
    torch.cuda.synchronize()
    print(f"rep {rep}: {e0.elapsed_time(e1):.3f} ms, {len(h)} levels", flush=True)
    h.close()
