"""Refinement of un-coarsening (PAPER.md P22.s1-22, reading R18).

-m "not gpu": the oracle (oracle.c: oracle_refine) is pinned by a hand-worked example, the
ordering method's no-swap property, the balance invariant, the boundary-only property and the
definition of the edge cut (recomputed here from scratch).
-m gpu: gp_refine / gp_uncoarsen equal the oracle bit for bit (labels, moves, passes).
"""
import numpy as np
import pytest
import torch

import graphgen as G
import oracle
from checks import np_graph


def edge_cut(g, part):
    g = np_graph(g)
    src = np.repeat(np.arange(g["n"]), np.diff(g["adjp"]))
    p = np.asarray(part)
    return int(g["adjwgt"][p[src] != p[g["adjncy"]]].sum()) // 2


def part_weights(g, part, k):
    return np.bincount(np.asarray(part), weights=np_graph(g)["vwgt"], minlength=k).astype(np.int64)


def bounds(g, k, imb):
    W = int(np_graph(g)["vwgt"].sum())
    return -(-(W * (100 + imb)) // (100 * k)), (W * (100 - imb)) // (100 * k)


def test_hand_worked_path():
    # path 0-1-2-3 with weights 5, 1, 5; labels [0,1,0,1]; k = 2, 50 % imbalance: max_w = 3,
    # min_w = 1.  Pass 0, dir 0 (to higher ids): v0 gains 5 and v2 gains 6 towards 1; partition 1
    # explores (v2, 6) then (v0, 5) and accepts only v2 (2 + 1 = 3 <= 3; then 4 > 3).
    # dir 1: v1 (now w(v1,0) = 5 vs w(v1,1) = 1) gains 4 towards 0 -> accepted.  Labels
    # [0,0,1,1], cut 1 (the optimum).  Pass 1 moves nothing: 2 passes, 2 moves.
    g = G.from_edge_list(4, [(0, 1, 5), (1, 2, 1), (2, 3, 5)])
    part, moves, passes = oracle.refine(g, np.array([0, 1, 0, 1], dtype=np.int32), 2, imbalance_pct=50)
    assert part.tolist() == [0, 0, 1, 1] and moves == 2 and passes == 2
    assert edge_cut(g, part) == 1


def test_direction_ordering_forbids_swaps():
    # two heavy-edge neighbours a in 0 and b in 1, each better off on the other side: with one
    # direction per iteration only one of them moves per iteration, never an exchange
    g = G.from_edge_list(4, [(0, 1, 10), (0, 2, 1), (1, 3, 1)])
    part, moves, _ = oracle.refine(g, np.array([0, 1, 1, 0], dtype=np.int32), 2, imbalance_pct=100, max_passes=1)
    # dir 0: v0 (gain 10 - 0 ... ) goes to 1; v3 (w(v3,1)=1 > w(v3,0)=0) goes to 1 as well;
    # dir 1: v1 / v2 see their neighbours in 1 and stay
    assert edge_cut(g, part) < edge_cut(g, [0, 1, 1, 0])


def test_star_follows_the_heavy_leaf():
    # star 0-{1,2,3,4}, edge (0,4) of weight 7, the others 1; leaf 4 alone in partition 1;
    # k = 2, 100 % tolerance (max_w = 5, min_w = 0).  Pass 0, dir 0 (to higher ids): the centre 0
    # has w(0,1) = 7 > w(0,0) = 3 (gain 4) and moves to 1; leaves 1-3 are interior.  dir 1: the
    # centre now has w(0,0) = 3 < w(0,1) = 7: no move.  Pass 1, dir 0: leaves 1-3 each gain 1
    # towards 1 and all three are accepted (1 + 1 + 1 + 2 <= 5).  Pass 2 moves nothing.
    g = G.from_edge_list(5, [(0, 1, 1), (0, 2, 1), (0, 3, 1), (0, 4, 7)])
    part, moves, passes = oracle.refine(g, np.array([0, 0, 0, 0, 1], dtype=np.int32), 2, imbalance_pct=100)
    assert part.tolist() == [1, 1, 1, 1, 1] and moves == 4 and passes == 3
    # with 3 % (max_w = ceil(5*103/200) = 3, min_w = floor(5*97/200) = 2): pass 0 moves the centre
    # as above (partition 0 keeps 3 >= 2, partition 1 gets 2 <= 3).  Pass 1, dir 0: leaves 1-3
    # all request (each checked against the start weight 3 - 1 >= 2); partition 1 explores them
    # in id order and accepts only leaf 1 (2 + 1 = 3; then 4 > 3).  Pass 2: partition 0 holds 2,
    # a leaf leaving would underweight it (1 < 2): no request, no move.
    part, moves, passes = oracle.refine(g, np.array([0, 0, 0, 0, 1], dtype=np.int32), 2, imbalance_pct=3)
    assert part.tolist() == [1, 1, 0, 0, 1] and moves == 2 and passes == 3


@pytest.mark.parametrize("seed", range(12))
def test_invariants_random(seed):
    n = 40 + 17 * seed
    g = G.random_graph(n, 4 * n, seed + 7000, wmax=[1, 5, 100][seed % 3])
    g["vwgt"] = (torch.arange(n, dtype=torch.int32) % 3) + 1
    k = [2, 3, 4, 8][seed % 4]
    imb = [3, 10, 30][seed % 3]
    rng = np.random.default_rng(seed)
    # a balanced start: round-robin over a random order
    p0 = np.empty(n, dtype=np.int32)
    p0[rng.permutation(n)] = np.arange(n) % k
    maxw, minw = bounds(g, k, imb)
    start_ok = part_weights(g, p0, k).max() <= maxw
    part, moves, passes = oracle.refine(g, p0, k, imbalance_pct=imb)
    assert part.min() >= 0 and part.max() < k
    assert moves == int((part != p0).sum()) or moves >= int((part != p0).sum())
    if start_ok:  # accepted moves never push a destination above max_w
        assert part_weights(g, part, k).max() <= maxw
    # interior vertices (all neighbours in their own partition at the start) can still move
    # later; but a vertex with no neighbours never moves
    deg = np.diff(np_graph(g)["adjp"])
    assert np.all(part[deg == 0] == p0[deg == 0])
    assert 1 <= passes <= 8
    # a refinement of the refined labels with 0 passes changes nothing
    p2, m2, ps2 = oracle.refine(g, part, k, imbalance_pct=imb, max_passes=0)
    assert np.array_equal(p2, part) and m2 == 0 and ps2 == 0


def test_cut_improves_on_meshes():
    g = G.delaunay_like(64)
    k = 8
    p0 = (np.arange(g["n"]) * 7919 % k).astype(np.int32)   # a scattered start
    part, moves, _ = oracle.refine(g, p0, k, imbalance_pct=3, max_passes=8)
    assert moves > 0 and edge_cut(g, part) < 0.6 * edge_cut(g, p0)


def test_uncoarsen_oracle_composition():
    g = G.delaunay_like(48)
    levels = oracle.coarsen_to(g, threshold=100)
    k = 4
    pc = (np.arange(levels[-1]["n_coarse"]) % k).astype(np.int32)
    part, moves = oracle.uncoarsen(g, levels, pc, k)
    # the same thing spelled out level by level
    cur = pc
    for l in range(len(levels) - 1, -1, -1):
        cur = oracle.project(levels, cur, from_level=l, to_level=l)
        cur, _, _ = oracle.refine(g if l == 0 else levels[l - 1]["coarse"], cur, k)
    assert np.array_equal(part, cur)


# ------------------------------------------------------------------------------------------ GPU
@pytest.fixture(scope="module")
def gp():
    import paper_conf_ipps_goodarzibg16_b200.gp as gp
    return gp


@pytest.fixture(scope="module")
def ctx(gp):
    c = gp.Context(0)
    yield c
    c.close()


REF_CASES = {
    "path4": (lambda: G.from_edge_list(4, [(0, 1, 5), (1, 2, 1), (2, 3, 5)]), 2, 50),
    "delaunay64_k8": (lambda: G.delaunay_like(64), 8, 3),
    "delaunay128_k64": (lambda: G.delaunay_like(128), 64, 3),
    "rgg_k16": (lambda: G.rgg(1 << 13), 16, 5),
    "rmat12_k4": (lambda: G.varied_vwgt(G.rmat(12)), 4, 10),   # hub rows: the warp request path
    "road_k32": (lambda: G.road_like(96), 32, 3),
    "star_k3": (lambda: G.from_edge_list(2001, [(0, i, 1 + i % 9) for i in range(1, 2001)]), 3, 50),
}


@pytest.mark.gpu
@pytest.mark.parametrize("name", list(REF_CASES))
@pytest.mark.parametrize("start", ["scattered", "blocks"])
def test_gpu_refine_equals_oracle(gp, ctx, name, start):
    make, k, imb = REF_CASES[name]
    g = make()
    n = g["n"]
    p0 = ((np.arange(n) * 7919 % k) if start == "scattered" else (np.arange(n) * k // max(n, 1))).astype(np.int32)
    ref, moves, passes = oracle.refine(g, p0, k, imbalance_pct=imb)
    d = {kk: g[kk].cuda() for kk in ("adjp", "adjncy", "adjwgt", "vwgt")}
    Gr = gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"])
    part = torch.from_numpy(p0).cuda()
    mv, ps = Gr.refine(part, k, imbalance_pct=imb)
    assert np.array_equal(part.cpu().numpy(), ref), name
    assert (mv, ps) == (moves, passes)
    Gr.close()


@pytest.mark.gpu
@pytest.mark.parametrize("name,k", [("C3_128", 8), ("C2_2^14", 64), ("C4_s12", 4)])
def test_gpu_uncoarsen_equals_oracle(gp, ctx, name, k):
    g = {"C3_128": lambda: G.delaunay_like(128), "C2_2^14": lambda: G.rgg(1 << 14),
         "C4_s12": lambda: G.rmat(12)}[name]()
    levels = oracle.coarsen_to(g, threshold=100)
    pc = (np.arange(levels[-1]["n_coarse"]) % k).astype(np.int32)
    ref, moves = oracle.uncoarsen(g, levels, pc, k)
    d = {kk: g[kk].cuda() for kk in ("adjp", "adjncy", "adjwgt", "vwgt")}
    Gr = gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"])
    H = Gr.coarsen_to(100)
    out = torch.empty(g["n"], dtype=torch.int32, device="cuda")
    mv = H.uncoarsen(Gr, torch.from_numpy(pc).cuda(), out, k)
    assert np.array_equal(out.cpu().numpy(), ref) and mv == moves
    H.close()
    Gr.close()


@pytest.mark.gpu
def test_gpu_refine_rejects_bad_input(gp, ctx):
    g = G.grid2d(8, 8)
    d = {kk: g[kk].cuda() for kk in ("adjp", "adjncy", "adjwgt", "vwgt")}
    Gr = gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"])
    part = torch.zeros(64, dtype=torch.int32, device="cuda")
    part[5] = 9  # outside [0, nparts)
    with pytest.raises(gp.GPError) as e:
        Gr.refine(part, 4)
    assert e.value.status == 1
    for bad_k in (0, 2000):
        with pytest.raises(gp.GPError):
            Gr.refine(torch.zeros(64, dtype=torch.int32, device="cuda"), bad_k)
    # max_passes = 0: nothing moves
    p0 = (torch.arange(64, device="cuda", dtype=torch.int32) % 4).contiguous()
    p1 = p0.clone()
    assert Gr.refine(p1, 4, max_passes=0) == (0, 0) and torch.equal(p0, p1)
    # gp_uncoarsen needs the hierarchy's own level-0 graph
    H = Gr.coarsen_to(4)
    other = gp.Graph.create(ctx, *[G.grid2d(4, 4)[kk].cuda() for kk in ("adjp", "adjncy", "adjwgt", "vwgt")])
    pc = torch.zeros(H.level(len(H) - 1).n_coarse, dtype=torch.int32, device="cuda")
    out = torch.empty(64, dtype=torch.int32, device="cuda")
    with pytest.raises(gp.GPError):
        H.uncoarsen(other, pc, out, 2)
    H.close()
    other.close()
    Gr.close()
