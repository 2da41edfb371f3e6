"""Projection (un-coarsening step 1): oracle pins (CPU) and GPU parity.

Pins of oracle.project, independent of its formula:
  * a hand-worked path (P6: M=[1,0,3,2,5,4], CM=[0,0,1,1,2,2]);
  * multilevel invariants (textbook): projecting a labelling of the coarsest graph down to
    level 0 preserves every part's total vertex weight (cvwgt sums the pair, P12.s27) and
    the edge cut (a collapsed edge is internal to one coarse vertex, a coarse edge weighs the
    sum of the fine edges between the two groups, P12.s28) -- checked on the fine graph
    itself, never through CM;
  * partners get the same label at every level.
"""
import numpy as np
import pytest
import torch

import graphgen as G
import oracle


def _np(g):
    return {k: (v.numpy() if hasattr(v, "numpy") else np.asarray(v)) for k, v in g.items()}


def _cut(g, part):
    adjp, adjncy, adjwgt = np.asarray(g["adjp"]), np.asarray(g["adjncy"]), np.asarray(g["adjwgt"])
    src = np.repeat(np.arange(len(adjp) - 1), np.diff(adjp))
    return int(adjwgt[part[src] != part[adjncy]].sum()) // 2


def _part_weights(vwgt, part, k):
    return np.bincount(part, weights=np.asarray(vwgt, dtype=np.float64), minlength=k).astype(np.int64)


def test_project_hand_worked_path():
    g = G.from_edge_list(6, [(0, 1, 1), (1, 2, 1), (2, 3, 1), (3, 4, 1), (4, 5, 1)])
    levels = oracle.coarsen_to(_np(g), threshold=3, max_levels=1)
    assert levels[0]["cmap"].tolist() == [0, 0, 1, 1, 2, 2]
    assert oracle.project(levels, [7, 8, 9]).tolist() == [7, 7, 8, 8, 9, 9]


@pytest.mark.parametrize("name,k", [("delaunay", 8), ("rgg", 16), ("rmat", 4), ("road", 64)])
def test_project_preserves_cut_and_part_weights(name, k):
    g = _np({"delaunay": lambda: G.delaunay_like(40), "rgg": lambda: G.rgg(3000),
             "rmat": lambda: G.rmat(10, 8), "road": lambda: G.road_like(60)}[name]())
    levels = oracle.coarsen_to(g, threshold=50)
    coarsest = levels[-1]["coarse"]
    rng = np.random.default_rng(5)
    pc = rng.integers(0, k, size=len(coarsest["vwgt"])).astype(np.int32)
    pf = oracle.project(levels, pc)
    assert len(pf) == len(g["vwgt"])
    assert np.array_equal(_part_weights(g["vwgt"], pf, k), _part_weights(coarsest["vwgt"], pc, k))
    assert _cut(g, pf) == _cut(coarsest, pc)
    # partial projections compose: coarsest -> level 2 -> level 0
    if len(levels) > 3:
        mid = oracle.project(levels, pc, to_level=2)
        assert np.array_equal(oracle.project(levels, mid, from_level=1), pf)


def test_project_partners_share_labels():
    g = _np(G.delaunay_like(32))
    levels = oracle.coarsen_to(g, threshold=20)
    ids = np.arange(len(levels[-1]["coarse"]["vwgt"]), dtype=np.int32)
    for to in range(len(levels)):
        lab = oracle.project(levels, ids, to_level=to)
        m = np.asarray(levels[to]["match"])
        assert np.array_equal(lab, lab[m])


@pytest.mark.gpu
@pytest.mark.parametrize("name", ["delaunay", "rmat", "grid"])
def test_gpu_project_equals_oracle(name):
    import paper_conf_ipps_goodarzibg16_b200.gp as gp
    from gpu_helpers import to_device

    g = _np({"delaunay": lambda: G.delaunay_like(300), "rmat": lambda: G.rmat(14, 8),
             "grid": lambda: G.grid2d(64, 64, unit=True)}[name]())
    ctx = gp.Context(0)
    d = to_device(g)
    graph = gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"])
    hier = graph.coarsen_to(100)
    levels = oracle.coarsen_to(g, threshold=100)
    assert len(hier) == len(levels)
    L = len(levels)
    rng = np.random.default_rng(1)
    for frm, to in [(L - 1, 0), (L - 1, L - 1), (L // 2, 1 if L > 2 else 0)]:
        nc = levels[frm]["n_coarse"]
        pc = rng.integers(0, 64, size=nc).astype(np.int32)
        out = torch.full((levels[to]["n"],), -5, dtype=torch.int32, device="cuda")
        hier.project(torch.from_numpy(pc).cuda(), out, from_level=frm, to_level=to)
        ref = oracle.project(levels, pc, from_level=frm, to_level=to)
        assert np.array_equal(out.cpu().numpy(), ref), (frm, to)
    hier.close()
    graph.close()
    ctx.close()
