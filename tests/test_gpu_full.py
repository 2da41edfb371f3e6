"""Full-size parity (-m gpu): BASELINE.json's configs at their full sizes, in the launch
configuration bench.py times (gp_coarsen_to on a device-resident graph).

C1, C2, C3 and C5 are compared with the oracle at every level, element by element.  C4
(R-MAT scale 24, 2^28 endpoint draws) is compared with the oracle on level 0 (matching,
cmap and coarse graph); its later levels are checked by the per-level invariants, which
hold at any size.
"""
import numpy as np
import pytest
import torch

import graphgen as G
import oracle
from checks import np_graph
from gpu_helpers import assert_levels_equal, gpu_coarsen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gp():
    import paper_conf_ipps_goodarzibg16_b200.gp as gp
    return gp


@pytest.fixture(scope="module")
def ctx(gp):
    c = gp.Context(0)
    yield c
    c.close()


def _host(g):
    return {k: (v.cpu() if isinstance(v, torch.Tensor) else v) for k, v in g.items()}


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3", "C5"])
def test_full_config_all_levels(gp, ctx, cfg):
    g = G.make_config(cfg, device="cuda")
    got = gpu_coarsen(gp, ctx, g, threshold=100)
    gh = _host(g)
    del g
    torch.cuda.empty_cache()
    ref = oracle.coarsen_to(gh, threshold=100)
    assert_levels_equal(got, ref, cfg)


def _vector_invariants(fine, lvl):
    """Vectorised per-level invariants for large graphs."""
    f = np_graph(fine)
    n = f["n"]
    m = lvl["match"].astype(np.int64)
    cm = lvl["cmap"].astype(np.int64)
    assert np.all(m[m] == np.arange(n))
    src = np.repeat(np.arange(n), np.diff(f["adjp"]))
    single = m == np.arange(n)
    assert not np.any(single[src] & single[f["adjncy"]]), "not maximal"
    matched = ~single
    # every matched pair is an edge: the arc (u, M[u]) exists
    is_pair_arc = m[src] == f["adjncy"]
    assert np.bincount(src[is_pair_arc], minlength=n)[matched].min(initial=1) == 1
    n_c = lvl["n_coarse"]
    lead = np.arange(n) <= m
    assert np.array_equal(cm[lead], np.arange(n_c)) and np.all(cm == cm[m])
    c = {k: lvl["coarse"][k].astype(np.int64) for k in ("adjp", "adjncy", "adjwgt", "vwgt")}
    assert c["vwgt"].sum() == f["vwgt"].sum()
    assert c["adjwgt"].sum() == f["adjwgt"].sum() - f["adjwgt"][is_pair_arc].sum()
    rows = np.repeat(np.arange(n_c), np.diff(c["adjp"]))
    assert not np.any(rows == c["adjncy"]), "coarse self-loop"
    same = rows[1:] == rows[:-1]
    assert np.all(np.diff(c["adjncy"])[same] > 0), "coarse rows not strictly increasing"
    # coarse symmetry with equal weights: sort the reversed arcs and compare
    fwd = rows * n_c + c["adjncy"]
    rev = c["adjncy"] * n_c + rows
    o = np.argsort(rev, kind="stable")
    assert np.array_equal(fwd, rev[o]) and np.array_equal(c["adjwgt"], c["adjwgt"][o])


def test_full_rmat_s24(gp, ctx):
    g = G.make_config("C4", device="cuda")
    got = gpu_coarsen(gp, ctx, g, threshold=100)
    gh = _host(g)
    del g
    torch.cuda.empty_cache()
    # level 0 against the oracle, element by element
    m, rounds, maximal = oracle.match_level(gh)
    assert rounds == got[0]["rounds"] and maximal == got[0]["maximal"]
    assert np.array_equal(m, got[0]["match"])
    cm, n_c = oracle.cmap(m)
    assert np.array_equal(cm, got[0]["cmap"]) and n_c == got[0]["n_coarse"]
    c = oracle.contract(gh, m, cm, n_c)
    for k in ("adjp", "adjncy", "adjwgt", "vwgt"):
        assert np.array_equal(c[k], got[0]["coarse"][k]), k
    # every level: invariants that hold at any size
    fine = gh
    for lvl in got:
        _vector_invariants(fine, lvl)
        fine = lvl["coarse"]
