"""C3 step time: level kernels only vs the partitioned tail (GP_PART), 8 reps each, alternating."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as G  # noqa: E402
import paper_conf_ipps_goodarzibg16_b200.gp as gp  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
ctx = gp.Context(0)
g = G.make_config(cfg, device="cuda")
graph = gp.Graph.create(ctx, g["adjp"], g["adjncy"], g["adjwgt"], g["vwgt"])
for setting in ("0", "1", "0", "1"):
    os.environ["GP_PART"] = setting
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
    print(f"{cfg} GP_PART={setting}: {sorted(ts)[len(ts)//2]:.3f} ms median, {nl} levels", flush=True)
