"""Small coarsen_to runs for compute-sanitizer (memcheck / racecheck / synccheck), each checked
bit for bit against the oracle so that a sanitizer run also proves the results:
    python scripts/sanitize_cases.py c3_256 | star5000 | loopback3 | c1_tail | medium_tail |
                                     part_tail | part_many | win | refine"""
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
elif case == "c1_tail":  # the coarse-level tail kernel (csrc/small.cu) runs every level of C1
    ctx, g, thr = gp.Context(0), G.make_config("C1"), 100
elif case == "medium_tail":  # the cluster tail (csrc/medium.cu): forced for a 16 K-vertex mesh
    os.environ["GP_SMALL"] = "0"
    os.environ["GP_MEDIUM"] = "1"
    ctx, g, thr = gp.Context(0), G.delaunay_like(128), 100
elif case == "part_tail":  # the partitioned grid tail (csrc/part.cu) for every level of a mesh
    os.environ["GP_SMALL"] = "0"
    ctx, g, thr = gp.Context(0), G.delaunay_like(128), 100
elif case == "part_many":  # ... on many CTAs with rows and window lookups from global memory
    os.environ["GP_SMALL"] = "0"
    os.environ["GP_PART_W"] = "256"
    os.environ["GP_PART_GARCS"] = "1"
    os.environ["GP_PART_WCAP"] = "64"
    ctx, g, thr = gp.Context(0), G.varied_vwgt(G.shuffle_rows(G.rmat(12), 3)), 10
elif case == "win":  # the opt-in windowed big-level matching (csrc/match_win.cu)
    os.environ["GP_WIN"] = "1"
    os.environ["GP_WIN_N"] = "2000"
    ctx, g, thr = gp.Context(0), G.delaunay_like(128), 100
elif case == "refine":  # gp_uncoarsen: projection + refinement kernels (csrc/refine.cu)
    import numpy as np
    import torch
    ctx, g = gp.Context(0), G.rmat(12)
    levels = oracle.coarsen_to(g, threshold=100)
    pc = (np.arange(levels[-1]["n_coarse"]) % 8).astype(np.int32)
    ref, moves = oracle.uncoarsen(g, levels, pc, 8)
    d = {k: g[k].cuda() for k in ("adjp", "adjncy", "adjwgt", "vwgt")}
    Gr = gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"])
    H = Gr.coarsen_to(100)
    out = torch.empty(g["n"], dtype=torch.int32, device="cuda")
    mv = H.uncoarsen(Gr, torch.from_numpy(pc).cuda(), out, 8)
    assert np.array_equal(out.cpu().numpy(), ref) and mv == moves
    print(f"refine: uncoarsen of {len(levels)} levels bit-exact vs the oracle ({mv} moves)")
    raise SystemExit(0)
else:
    raise SystemExit(f"unknown case {case}")
got = gpu_coarsen(gp, ctx, g, threshold=thr)
assert_levels_equal(got, oracle.coarsen_to(g, threshold=thr), case)
print(f"{case}: {len(got)} levels bit-exact vs the oracle")
