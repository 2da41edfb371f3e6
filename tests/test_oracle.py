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
from checks import (check_csr, check_level, check_matching, contract_by_sparse_triple_product, one_shot_hem,
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


# ---- stop-rule boundaries (readings R12 / R13) ------------------------------------------
# R12 "coarsen until |V| is below a threshold" (P10.s16, P20.s30) is read as "continue while
# n > threshold"; R13 (Metis' "difference ... less than a threshold", P12.s30) as "stop after a
# level with 100*n_c > 95*n".  Each case sits exactly on a boundary, so the strict and the
# non-strict comparison give different level counts (a '>=' in either test fails a case).

def test_threshold_boundary_c1_closed_form():
    # C1's closed form: n = 4096 -> 2048 -> ... -> 64, one halving per level
    g = G.make_config("C1")
    lv = oracle.coarsen_to(g, threshold=64)
    assert [l["n"] for l in lv] == [4096, 2048, 1024, 512, 256, 128]       # n == 64 is not > 64: stop
    assert lv[-1]["n_coarse"] == 64 and lv[-1]["stop_reason"] == oracle.STOP_THRESHOLD
    lv = oracle.coarsen_to(g, threshold=63)                                  # 64 > 63: one more level
    assert [l["n"] for l in lv][-1] == 64 and lv[-1]["n_coarse"] == 32
    lv = oracle.coarsen_to(g, threshold=4096)                                # input already at the threshold
    assert lv == []


def test_stall_boundary_one_edge():
    # 20 vertices, one edge: level 0 gives n_c = 19 and 100*19 == 95*20 -- not a stall
    # (strict '>'); level 1 has no edge, n_c = n = 19 -> stall.  So exactly 2 levels.
    g = G.from_edge_list(20, [(3, 11, 5)])
    lv = oracle.coarsen_to(g, threshold=1)
    assert [(l["n"], l["n_coarse"]) for l in lv] == [(20, 19), (19, 19)]
    assert [l["stop_reason"] for l in lv] == [0, oracle.STOP_STALL]
    # 21 vertices, one edge: 100*20 = 2000 > 95*21 = 1995 -> stall after level 0
    g = G.from_edge_list(21, [(3, 11, 5)])
    lv = oracle.coarsen_to(g, threshold=1)
    assert [(l["n"], l["n_coarse"]) for l in lv] == [(21, 20)]
    assert lv[0]["stop_reason"] == oracle.STOP_STALL
    # stall_ratio_pct is the percentage of the same integer test: 100*19 > 94*20 stalls at once
    g = G.from_edge_list(20, [(3, 11, 5)])
    lv = oracle.coarsen_to(g, threshold=1, stall_ratio_pct=94)
    assert len(lv) == 1 and lv[0]["stop_reason"] == oracle.STOP_STALL


def test_max_levels_boundary():
    g = G.make_config("C1")
    lv = oracle.coarsen_to(g, threshold=100, max_levels=3)
    assert len(lv) == 3 and lv[-1]["stop_reason"] == oracle.STOP_MAX_LEVELS
    lv = oracle.coarsen_to(g, threshold=100, max_levels=6)                  # the 6th level also reaches 64
    assert len(lv) == 6 and lv[-1]["stop_reason"] == oracle.STOP_THRESHOLD


# ---- the paper's one-shot matching ----------------------------------
# P18.s7-13: ONE lock-free HEM pass (every vertex grabs its heaviest neighbour) + the conflict
# kernel (non-mutual choices self-match).  With the races removed and ties to the lower id,
# that is exactly the pinned rule capped at one round (max_rounds = 1, leftover = the conflict
# kernel's self-matches).  checks.one_shot_hem computes it directly from the graph.
@pytest.mark.parametrize("seed", range(30))
def test_one_shot_equals_max_rounds_1(seed):
    n = 10 + 37 * seed
    g = G.random_graph(n, 3 * n, seed + 4000, wmax=[1, 3, 100][seed % 3])
    m, rounds, maximal = oracle.match_level(g, max_rounds=1)
    ref = one_shot_hem(g)
    assert np.array_equal(m.astype(np.int64), ref)
    assert rounds == (1 if np.any(ref != np.arange(n)) else 0)


@pytest.mark.parametrize("name,make", [("C3", lambda: G.delaunay_like(64)), ("C5", lambda: G.road_like(64)),
                                       ("C2", lambda: G.rgg(1 << 12)), ("C4", lambda: G.rmat(10))])
def test_one_shot_hierarchy(name, make):
    g = make()
    levels = oracle.coarsen_to(g, threshold=100, max_rounds=1)
    cur = g
    for l in levels:
        assert np.array_equal(l["match"].astype(np.int64), one_shot_hem(cur))
        check_matching(cur, l["match"], maximal=False)
        cur = l["coarse"]
