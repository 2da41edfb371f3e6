"""Full-size parity (-m gpu): BASELINE.json's configs at their full sizes, in the launch
configuration bench.py times (gp_coarsen_to on a device-resident graph).

Every config is compared with the oracle at every level, element by element.  C4 (R-MAT
scale 24, 2^28 endpoint draws) chains the oracle's per-level functions level by level on the
already-verified coarse graphs, and also checks the per-level invariants.
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


_C4 = {}  # level inputs and GPU results, inherited by the forked verifier processes


def _verify_c4_level(i):
    """Oracle step of level i on level i-1's GPU coarse graph (already compared by the worker of
    level i-1); no CUDA in this (forked) process."""
    fine, lvl, last = _C4["inputs"][i], _C4["got"][i], _C4["last"]
    where = f"C4 level {i}"
    try:
        assert lvl["n"] == len(fine["adjp"]) - 1, where
        m, rounds, maximal = oracle.match_level(fine)
        assert rounds == lvl["rounds"] and maximal == lvl["maximal"], (where, rounds, lvl["rounds"])
        assert np.array_equal(m, lvl["match"]), f"{where}: match"
        cm, n_c = oracle.cmap(m)
        assert np.array_equal(cm, lvl["cmap"]) and n_c == lvl["n_coarse"], f"{where}: cmap"
        c = oracle.contract(fine, m, cm, n_c)
        for k in ("adjp", "adjncy", "adjwgt", "vwgt"):
            assert np.array_equal(c[k], lvl["coarse"][k]), f"{where}: coarse {k}"
        stall = 100 * n_c > 95 * lvl["n"]
        if i < last:
            assert lvl["stop_reason"] == 0 and not stall and n_c > 100, where
        else:
            assert lvl["stop_reason"] == (oracle.STOP_STALL if stall else oracle.STOP_THRESHOLD), where
        return i, ""
    except AssertionError as e:
        return i, f"{where}: {e}"


def test_full_rmat_s24(gp, ctx):
    """C4 at full size, EVERY level bit-compared with the oracle.  Level l's oracle step
    (match_level, cmap, contract) runs on level l-1's GPU coarse graph; together the levels
    are the oracle's own hierarchy, because each level's input is itself proven equal to the
    oracle's by the check of the level before.  The levels are checked in parallel processes
    (one oracle level of R-MAT s24 is minutes of single-threaded C)."""
    import multiprocessing as mp
    g = G.make_config("C4", device="cuda")
    got = gpu_coarsen(gp, ctx, g, threshold=100)
    gh = {k: np.asarray(v.cpu()) if isinstance(v, torch.Tensor) else v for k, v in g.items()}
    del g
    torch.cuda.empty_cache()
    _C4["inputs"] = [gh] + [lvl["coarse"] for lvl in got[:-1]]
    _C4["got"] = got
    _C4["last"] = len(got) - 1
    with mp.get_context("fork").Pool(len(got)) as pool:
        res = pool.map(_verify_c4_level, range(len(got)))
    bad = [msg for _, msg in res if msg]
    assert not bad, bad
    _vector_invariants(_C4["inputs"][-1], got[-1])  # (implied by the bit-exact levels; cheap on the last)
