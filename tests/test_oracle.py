"""Pins of the C oracle against what the paper and mathematics fix (-m "not gpu").

Each pin is chosen so a plausible mistake fails one of them:
  * golden hand-worked graphs (tests/golden/hand_worked.json): a wrong tie rule, a
    transposed leader test, a dropped weight sum or a kept self-loop changes an array;
  * textbook greedy matching under the strict edge order (independent code in checks.py);
  * brute force on <= 10 vertices: maximality (P12.s21) and w(M) >= max w / 2;
  * contraction == off-diagonal of P^T A P, P^T vwgt (scipy.sparse, P12.s26-28);
  * closed form of config C1 (tests/golden/c1_closed_form.json);
  * unit paths take floor(n/2) rounds; invariants after every level; neighbour-order
    independence (R15).
"""
import json
import os

import numpy as np
import pytest
import torch

import graphgen as G
import oracle
from checks import (check_csr, check_level, check_matching, contract_by_sparse_triple_product,
                    edge_list, greedy_matching, max_weight_matching_bruteforce, np_graph)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _golden_cases():
    with open(os.path.join(GOLDEN, "hand_worked.json")) as f:
        return json.load(f)["cases"]


@pytest.mark.parametrize("case", _golden_cases(), ids=lambda c: c["name"])
def test_golden_hand_worked(case):
    g = G.from_edge_list(case["n"], case["edges"])
    m, rounds, maximal = oracle.match_level(g)
    assert maximal
    assert rounds == case["rounds"]
    assert m.tolist() == case["match"]
    cm, n_c = oracle.cmap(m)
    assert n_c == case["n_coarse"]
    assert cm.tolist() == case["cmap"]
    c = oracle.contract(g, m, cm, n_c)
    for k in ("adjp", "adjncy", "adjwgt", "vwgt"):
        assert c[k].tolist() == case["coarse"][k], k


def test_c1_closed_form():
    with open(os.path.join(GOLDEN, "c1_closed_form.json")) as f:
        ref = json.load(f)
    g = G.make_config("C1")
    levels = oracle.coarsen_to(g, threshold=100)
    assert [l["n"] for l in levels] + [levels[-1]["n_coarse"]] == ref["n"]
    assert [l["nnz"] // 2 for l in levels] + [levels[-1]["coarse"]["nnz"] // 2] == ref["edges"]
    wsum = [int(np_graph(g)["adjwgt"].sum()) // 2] + [int(l["coarse"]["adjwgt"].astype(np.int64).sum()) // 2
                                                      for l in levels]
    assert wsum == ref["edge_weight_sum"]
    assert [l["rounds"] for l in levels] == ref["rounds"]
    last = levels[-1]["coarse"]
    assert set(last["vwgt"].tolist()) == {ref["final_vwgt"]}
    assert set(last["adjwgt"].tolist()) == {ref["final_edge_weight"]}
    assert levels[-1]["stop_reason"] == oracle.STOP_THRESHOLD


@pytest.mark.parametrize("n", list(range(1, 21)))
def test_unit_path_rounds(n):
    g = G.from_edge_list(n, [(i, i + 1, 1) for i in range(n - 1)])
    m, rounds, _ = oracle.match_level(g)
    assert rounds == n // 2
    assert m.tolist() == [i ^ 1 if (i ^ 1) < n else i for i in range(n)]


def _random_cases():
    cases = []
    for seed in range(60):
        n = 5 + (seed * 7) % 60
        m = n * (1 + seed % 5)
        wmax = [1, 2, 3, 100][seed % 4]
        cases.append((n, m, seed, wmax))
    return cases


@pytest.mark.parametrize("n,m,seed,wmax", _random_cases())
def test_equals_greedy_matching(n, m, seed, wmax):
    g = G.random_graph(n, m, seed, wmax)
    mo, rounds, maximal = oracle.match_level(g)
    assert maximal
    ref = greedy_matching(n, edge_list(g))
    assert np.array_equal(mo.astype(np.int64), ref)


@pytest.mark.parametrize("seed", range(150))
def test_bruteforce_small(seed):
    n = 2 + seed % 9                                       # 2..10 vertices
    g = G.random_graph(n, 2 * n, seed + 500, wmax=[1, 3, 10][seed % 3])
    m, _, maximal = oracle.match_level(g)
    assert maximal
    check_matching(g, m, maximal=True)
    edges = edge_list(g)
    wm = sum(w for u, v, w in edges if m[u] == v)
    best = max_weight_matching_bruteforce(n, edges)
    assert 2 * wm >= best


@pytest.mark.parametrize("seed", range(25))
def test_contraction_equals_sparse_triple_product(seed):
    n = 20 + 13 * seed
    g = G.random_graph(n, 3 * n, seed + 900, wmax=[1, 5, 100][seed % 3])
    g["vwgt"] = (torch.arange(n, dtype=torch.int32) % 7) + 1
    m, _, _ = oracle.match_level(g)
    cm, n_c = oracle.cmap(m)
    c = oracle.contract(g, m, cm, n_c)
    ref = contract_by_sparse_triple_product(g, cm, n_c)
    for k in ("adjp", "adjncy", "adjwgt", "vwgt"):
        assert np.array_equal(c[k].astype(np.int64), ref[k]), k
    check_level(g, m, cm, n_c, c)


def test_cmap_definition_literal():
    # cmap of a hand-made matching, checked against P18.s16-27 read as "coarse id = rank of
    # the leader among leaders in id order; partner copies its leader's id" (R7)
    match = np.array([3, 1, 4, 0, 2, 5], dtype=np.int32)
    cm, n_c = oracle.cmap(match)
    assert n_c == 4
    assert cm.tolist() == [0, 1, 2, 0, 2, 3]


def test_max_rounds_cap():
    g = G.grid2d(8, 8)
    m_full, r_full, maximal = oracle.match_level(g)
    assert maximal and r_full > 2
    m2, r2, maximal2 = oracle.match_level(g, max_rounds=2)
    assert r2 == 2 and not maximal2
    check_matching(g, m2, maximal=False)


def test_empty_and_isolated():
    g = G.from_edge_list(0, [])
    m, r, _ = oracle.match_level(g)
    assert len(m) == 0 and r == 0
    g = G.from_edge_list(5, [])
    m, r, mx = oracle.match_level(g)
    assert m.tolist() == list(range(5)) and r == 0 and mx
    levels = oracle.coarsen_to(g, threshold=1)
    assert len(levels) == 1 and levels[0]["stop_reason"] == oracle.STOP_STALL


SMALL_CONFIGS = [("C2", lambda: G.rgg(1 << 12)), ("C3", lambda: G.delaunay_like(64)),
                 ("C4", lambda: G.rmat(10)), ("C5", lambda: G.road_like(96)),
                 ("C4unit", lambda: G.rmat(9, unit=True))]


@pytest.mark.parametrize("name,make", SMALL_CONFIGS, ids=[c[0] for c in SMALL_CONFIGS])
def test_coarsen_invariants_small_configs(name, make):
    g = make()
    check_csr(g, name)
    levels = oracle.coarsen_to(g, threshold=100)
    cur = g
    for l in levels:
        check_matching(cur, l["match"], maximal=True)
        check_level(cur, l["match"], l["cmap"], l["n_coarse"], l["coarse"])
        cur = l["coarse"]
    last = levels[-1]
    assert last["stop_reason"] in (oracle.STOP_THRESHOLD, oracle.STOP_STALL)
    if last["stop_reason"] == oracle.STOP_STALL:
        assert 100 * last["n_coarse"] > 95 * last["n"]
    for l in levels[:-1]:
        assert 100 * l["n_coarse"] <= 95 * l["n"] and l["n"] > 100


@pytest.mark.parametrize("seed", range(8))
def test_neighbour_order_independence(seed):
    g = G.rgg(1 << 10)
    gn = np_graph(g)
    rng = np.random.default_rng(seed)
    adjncy = gn["adjncy"].copy()
    adjwgt = gn["adjwgt"].copy()
    for u in range(gn["n"]):
        a, b = gn["adjp"][u], gn["adjp"][u + 1]
        p = rng.permutation(b - a) + a
        adjncy[a:b] = adjncy[p]
        adjwgt[a:b] = adjwgt[p]
    h = dict(gn, adjncy=adjncy, adjwgt=adjwgt)
    la = oracle.coarsen_to(g, 100)
    lb = oracle.coarsen_to(h, 100)
    assert len(la) == len(lb)
    for x, y in zip(la, lb):
        assert np.array_equal(x["match"], y["match"]) and x["rounds"] == y["rounds"]
        for k in ("adjp", "adjncy", "adjwgt", "vwgt"):
            assert np.array_equal(x["coarse"][k], y["coarse"][k])


def test_relabel_equivariance_distinct_weights():
    # with all-distinct weights the tie rule never fires, so relabelling vertices maps the
    # matched pair set accordingly
    n = 200
    g = G.random_graph(n, 800, 77, wmax=1 << 30)
    edges = edge_list(g)
    ws = [w for _, _, w in edges]
    if len(set(ws)) != len(ws):
        pytest.skip("weight collision")
    perm = np.random.default_rng(3).permutation(n)
    h = G.from_edge_list(n, [(int(perm[u]), int(perm[v]), w) for u, v, w in edges])
    ma, _, _ = oracle.match_level(g)
    mb, _, _ = oracle.match_level(h)
    assert np.array_equal(perm[ma], mb[perm])
