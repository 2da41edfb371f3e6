"""Sharded path (-m gpu): gp_coarsen_to over G ranks equals the oracle bit for bit.

The loopback context runs G simulated ranks on one GPU: every rank has private buffers and
every exchange (round all-gathers of boundary proposals, leader-count / CM all-gathers,
partner-row send/recv) is a device copy between them, with the same kernels, buffers and
layouts as the NCCL transport (csrc/dist.cu).  So a protocol bug (a missing ghost value, a
wrong rank offset, a lost shipped row) shows up here as a mismatch against the oracle.
Shard boundaries cut through rows, matched pairs and hub rows; G up to 8.

Folding: once the coarse graph has at most GP_FOLD_N vertices
every rank gathers it and finishes on the single-GPU pipeline.  Each case runs with folding
off (every level sharded), with the default limit (fold right after level 0 on these sizes) and
with a limit a few levels down (sharded levels, then the folded rest).
"""
import numpy as np
import pytest
import torch

import graphgen as G
import oracle
from checks import check_level
from gpu_helpers import assert_levels_equal, gpu_coarsen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gp():
    import paper_conf_ipps_goodarzibg16_b200.gp as gp
    return gp


_ctxs = {}


def _ctx(gp, nranks):
    if nranks not in _ctxs:
        _ctxs[nranks] = gp.Context(0, loopback=nranks)
    return _ctxs[nranks]


def _host(g):
    return {k: (v.cpu() if isinstance(v, torch.Tensor) else v) for k, v in g.items()}


GRAPHS = {
    "grid32": lambda: G.grid2d(32, 32, unit=True),
    "delaunay64": lambda: G.delaunay_like(64),
    "rgg4k": lambda: G.rgg(4096),
    "road96": lambda: G.road_like(96),
    "rmat12": lambda: G.rmat(12, 8),
    "rmat10_unit": lambda: G.rmat(10, 8, unit=True),
    "random": lambda: G.random_graph(3000, 12000, seed=7),
}


FOLDS = ["off", "default", "mid"]


def _set_fold(monkeypatch, fold, n):
    # GP_FOLD_N is read by the library on every gp_coarsen_to call
    if fold == "off":
        monkeypatch.setenv("GP_FOLD_N", "0")
    elif fold == "mid":
        monkeypatch.setenv("GP_FOLD_N", str(max(1, n // 6)))
    else:
        monkeypatch.delenv("GP_FOLD_N", raising=False)


@pytest.mark.parametrize("fold", FOLDS)
@pytest.mark.parametrize("nranks", [2, 3, 4, 8])
@pytest.mark.parametrize("name", list(GRAPHS))
def test_loopback_hierarchy_equals_oracle(gp, name, nranks, fold, monkeypatch):
    g = _host(GRAPHS[name]())
    _set_fold(monkeypatch, fold, g["n"])
    ref = oracle.coarsen_to(g, threshold=20)
    got = gpu_coarsen(gp, _ctx(gp, nranks), g, threshold=20)
    assert_levels_equal(got, ref, f"{name} G={nranks} fold={fold}")


@pytest.mark.parametrize("fold", FOLDS)
@pytest.mark.parametrize("nranks", [2, 5])
def test_loopback_max_rounds_cap(gp, nranks, fold, monkeypatch):
    g = _host(G.delaunay_like(48))
    _set_fold(monkeypatch, fold, g["n"])
    ref = oracle.coarsen_to(g, threshold=20, max_rounds=2)
    got = gpu_coarsen(gp, _ctx(gp, nranks), g, threshold=20, max_rounds=2)
    assert_levels_equal(got, ref, f"cap G={nranks} fold={fold}")


@pytest.mark.parametrize("fold", FOLDS)
def test_loopback_max_levels_across_the_fold(gp, fold, monkeypatch):
    # the folded pipeline continues the level count (max_levels binds across the fold)
    g = _host(G.delaunay_like(64))
    _set_fold(monkeypatch, fold, g["n"])
    for ml in (1, 2, 3, 5):
        ref = oracle.coarsen_to(g, threshold=20, max_levels=ml)
        got = gpu_coarsen(gp, _ctx(gp, 4), g, threshold=20, max_levels=ml)
        assert_levels_equal(got, ref, f"max_levels={ml} fold={fold}")


@pytest.mark.parametrize("fold", FOLDS)
def test_loopback_more_ranks_than_coarse_vertices(gp, fold, monkeypatch):
    # ranks end up with empty shards at the coarse levels (and at level 0: 6 vertices, 8 ranks)
    g = _host(G.from_edge_list(6, [(0, 1, 1), (1, 2, 1), (2, 3, 1), (3, 4, 1), (4, 5, 1)]))
    _set_fold(monkeypatch, fold, g["n"])
    ref = oracle.coarsen_to(g, threshold=1)
    got = gpu_coarsen(gp, _ctx(gp, 8), g, threshold=1)
    assert_levels_equal(got, ref, f"path6 G=8 fold={fold}")


@pytest.mark.parametrize("fold", FOLDS)
def test_loopback_rm_ties_across_the_fold(gp, fold, monkeypatch):
    # the RM tie priority (R17) is a per-call option the folded pipeline inherits
    g = _host(G.rmat(11, 8, unit=True))
    _set_fold(monkeypatch, fold, g["n"])
    seed = 0x9E3779B9
    ref = oracle.coarsen_to(g, threshold=20, tie_seed=seed)
    got = gpu_coarsen(gp, _ctx(gp, 3), g, threshold=20, tie_seed=seed)
    assert_levels_equal(got, ref, f"rm fold={fold}")


def test_loopback_level_invariants_c3_quarter(gp, monkeypatch):
    # a 1024^2 Delaunay-like mesh over 4 ranks: every level satisfies the invariants and the
    # first level equals the oracle; folding (default limit: after level 1) gives the same
    # hierarchy as the fully sharded run, with far fewer launches (no per-round protocol)
    g = _host(G.delaunay_like(1024))
    ctx = _ctx(gp, 4)
    runs = {}
    for fold in ("off", "default"):
        _set_fold(monkeypatch, fold, g["n"])
        before = ctx.launch_count()
        runs[fold] = gpu_coarsen(gp, ctx, g, threshold=100)
        runs[fold + "_launches"] = ctx.launch_count() - before
    got = runs["default"]
    assert_levels_equal(got, runs["off"], "fold default vs off")
    assert runs["default_launches"] < runs["off_launches"]
    ref0 = oracle.coarsen_to(g, threshold=100, max_levels=1)[0]
    assert np.array_equal(got[0]["match"], ref0["match"])
    assert np.array_equal(got[0]["cmap"], ref0["cmap"])
    fine = {k: np.asarray(g[k]) for k in ("adjp", "adjncy", "adjwgt", "vwgt")}
    for lvl in got:
        check_level(fine, lvl["match"], lvl["cmap"], lvl["n_coarse"], lvl["coarse"])
        fine = lvl["coarse"]
