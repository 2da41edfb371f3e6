"""Sharded path (-m gpu): gp_coarsen_to over G ranks equals the oracle bit for bit.

The loopback context runs G simulated ranks on one GPU: every rank has private buffers and
every exchange (round all-gathers of boundary proposals, leader-count / CM all-gathers,
partner-row send/recv) is a device copy between them, with the same kernels, buffers and
layouts as the NCCL transport (csrc/dist.cu).  So a protocol bug (a missing ghost value, a
wrong rank offset, a lost shipped row) shows up here as a mismatch against the oracle.
Shard boundaries cut through rows, matched pairs and hub rows; G up to 8.
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


@pytest.mark.parametrize("nranks", [2, 3, 4, 8])
@pytest.mark.parametrize("name", list(GRAPHS))
def test_loopback_hierarchy_equals_oracle(gp, name, nranks):
    g = _host(GRAPHS[name]())
    ref = oracle.coarsen_to(g, threshold=20)
    got = gpu_coarsen(gp, _ctx(gp, nranks), g, threshold=20)
    assert_levels_equal(got, ref, f"{name} G={nranks}")


@pytest.mark.parametrize("nranks", [2, 5])
def test_loopback_max_rounds_cap(gp, nranks):
    g = _host(G.delaunay_like(48))
    ref = oracle.coarsen_to(g, threshold=20, max_rounds=2)
    got = gpu_coarsen(gp, _ctx(gp, nranks), g, threshold=20, max_rounds=2)
    assert_levels_equal(got, ref, f"cap G={nranks}")


def test_loopback_more_ranks_than_coarse_vertices(gp):
    # ranks end up with empty shards at the coarse levels (and at level 0: 6 vertices, 8 ranks)
    g = _host(G.from_edge_list(6, [(0, 1, 1), (1, 2, 1), (2, 3, 1), (3, 4, 1), (4, 5, 1)]))
    ref = oracle.coarsen_to(g, threshold=1)
    got = gpu_coarsen(gp, _ctx(gp, 8), g, threshold=1)
    assert_levels_equal(got, ref, "path6 G=8")


def test_loopback_level_invariants_c3_quarter(gp):
    # a 1024^2 Delaunay-like mesh over 4 ranks: every level satisfies the invariants and the
    # first level equals the oracle
    g = _host(G.delaunay_like(1024))
    got = gpu_coarsen(gp, _ctx(gp, 4), g, threshold=100)
    ref0 = oracle.coarsen_to(g, threshold=100, max_levels=1)[0]
    assert np.array_equal(got[0]["match"], ref0["match"])
    assert np.array_equal(got[0]["cmap"], ref0["cmap"])
    fine = {k: np.asarray(g[k]) for k in ("adjp", "adjncy", "adjwgt", "vwgt")}
    for lvl in got:
        check_level(fine, lvl["match"], lvl["cmap"], lvl["n_coarse"], lvl["coarse"])
        fine = lvl["coarse"]
