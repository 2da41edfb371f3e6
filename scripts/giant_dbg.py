"""Repeated coarsen_to on R-MAT with the grid-wide giant-row merge vs without (GP_GIANT_ROW=0)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen as G  # noqa: E402
import paper_conf_ipps_goodarzibg16_b200.gp as gp  # noqa: E402

arg = sys.argv[1] if len(sys.argv) > 1 else "20"
ctx = gp.Context(0)
g = G.make_config(arg, device="cuda") if arg.startswith("C") else G.rmat(int(arg), wmax=4, device="cuda")
graph = gp.Graph.create(ctx, g["adjp"], g["adjncy"], g["adjwgt"], g["vwgt"])


def run(giant):
    os.environ["GP_GIANT_ROW"] = str(giant)
    h = graph.coarsen_to(100)
    out = []
    for i in range(len(h)):
        m, c = h.download_level(i)
        co = h.download_coarse(i)
        out.append((m.numpy().copy(), c.numpy().copy(), {k: co[k].numpy().copy() for k in ("adjp", "adjncy", "adjwgt")}))
    h.close()
    torch.cuda.synchronize()
    return out


ref = run(0)
print("reference levels", len(ref), flush=True)
for rep in range(3):
    got = run(int(sys.argv[2]) if len(sys.argv) > 2 else 65536)
    same = len(got) == len(ref) and all(np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1]) and
                                         all(np.array_equal(a[2][k], b[2][k]) for k in a[2]) for a, b in zip(got, ref))
    print(f"rep {rep}: {len(got)} levels, identical to the per-CTA path: {same}", flush=True)
