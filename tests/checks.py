"""Independent checkers used by the tests (test infrastructure).

Nothing here calls the oracle or the CUDA path: these are the definitions the paper
and mathematics fix, written separately so that they can pin both.
"""
from __future__ import annotations

import itertools
from typing import Dict, List, Tuple

import numpy as np


def np_graph(g: Dict) -> Dict:
    out = {}
    for k in ("adjp", "adjncy", "adjwgt", "vwgt"):
        a = g[k]
        if hasattr(a, "numpy"):
            a = a.detach().cpu().numpy()
        out[k] = np.asarray(a, dtype=np.int64)
    out["n"] = len(out["adjp"]) - 1
    return out


def edge_list(g: Dict) -> List[Tuple[int, int, int]]:
    """Unique undirected edges (u < v, w) of a CSR graph."""
    g = np_graph(g)
    out = []
    for u in range(g["n"]):
        for j in range(g["adjp"][u], g["adjp"][u + 1]):
            v = int(g["adjncy"][j])
            if u < v:
                out.append((u, v, int(g["adjwgt"][j])))
    return out


def greedy_matching(n: int, edges: List[Tuple[int, int, int]]) -> np.ndarray:
    """Textbook sequential greedy matching: edges sorted by (w desc, min id asc, max id asc),
    take an edge iff both endpoints are free; unmatched vertices are self-matched.
    (The 1/2-approximation of maximum-weight matching; DESIGN.md §2.2 explains why the
    pinned handshake rule must equal it.)"""
    m = np.full(n, -1, dtype=np.int64)
    for u, v, w in sorted(edges, key=lambda e: (-e[2], min(e[0], e[1]), max(e[0], e[1]))):
        if m[u] < 0 and m[v] < 0:
            m[u] = v
            m[v] = u
    for u in range(n):
        if m[u] < 0:
            m[u] = u
    return m


def one_shot_hem(g: Dict) -> np.ndarray:
    """The paper's one-pass GPU matching with its races removed (P18.s7-13): every vertex
    takes its heaviest neighbour -- all vertices are unmatched when the single HEM kernel runs;
    ties go to the lower id (north_star) -- and the conflict kernel keeps a pair only if the
    choice is mutual ("M[u] = v and M[v] != u => M[u] = u", P18.s11-12); every other vertex is
    matched to itself.  Vectorised numpy, written from the definition (no rounds, no lists)."""
    g = np_graph(g)
    n = g["n"]
    m = np.arange(n, dtype=np.int64)
    if len(g["adjncy"]) == 0:
        return m
    src = np.repeat(np.arange(n), np.diff(g["adjp"]))
    # heaviest neighbour of every row: sort arcs by (row, -w, v) and take each row's first
    order = np.lexsort((g["adjncy"], -g["adjwgt"], src))
    first = np.ones(len(order), dtype=bool)
    first[1:] = src[order][1:] != src[order][:-1]
    pick = order[first]
    h = np.full(n, -1, dtype=np.int64)
    h[src[pick]] = g["adjncy"][pick]
    has = h >= 0
    mutual = np.zeros(n, dtype=bool)
    mutual[has] = h[h[has]] == np.arange(n)[has]
    m[mutual] = h[mutual]
    return m


def max_weight_matching_bruteforce(n: int, edges: List[Tuple[int, int, int]]) -> int:
    """Exhaustive maximum matching weight (tiny graphs only)."""
    best = 0
    adj = sorted(edges)

    def rec(i, used, acc):
        nonlocal best
        if acc > best:
            best = acc
        for k in range(i, len(adj)):
            u, v, w = adj[k]
            if not (used >> u) & 1 and not (used >> v) & 1:
                rec(k + 1, used | (1 << u) | (1 << v), acc + w)

    rec(0, 0, 0)
    return best


def check_csr(g: Dict, name: str = "graph") -> None:
    """Input contract (R15): adjp monotone from 0, ids in range, no self-loops,
    no duplicate arcs, symmetric with equal weights, weights >= 1."""
    g = np_graph(g)
    n = g["n"]
    adjp, adjncy, adjwgt = g["adjp"], g["adjncy"], g["adjwgt"]
    assert adjp[0] == 0 and np.all(np.diff(adjp) >= 0), name
    assert adjp[-1] == len(adjncy) == len(adjwgt), name
    assert len(g["vwgt"]) == n and np.all(g["vwgt"] >= 1), name
    if len(adjncy) == 0:
        return
    assert adjncy.min() >= 0 and adjncy.max() < n, name
    assert adjwgt.min() >= 1, name
    src = np.repeat(np.arange(n), np.diff(adjp))
    assert not np.any(src == adjncy), f"{name}: self-loop"
    key = src * n + adjncy
    assert len(np.unique(key)) == len(key), f"{name}: duplicate arc"
    fwd = dict(zip(key.tolist(), adjwgt.tolist()))
    rev = (adjncy * n + src).tolist()
    for k, r in zip(key.tolist(), rev):
        assert fwd.get(r) == fwd[k], f"{name}: asymmetric arc"


def check_matching(g: Dict, match: np.ndarray, maximal: bool = True) -> None:
    """M[M[u]] = u; M[u] != u => (u, M[u]) in E; maximality (P12.s20-21)."""
    g = np_graph(g)
    n = g["n"]
    m = np.asarray(match, dtype=np.int64)
    assert len(m) == n
    assert np.all(m[m] == np.arange(n)), "M[M[u]] != u"
    src = np.repeat(np.arange(n), np.diff(g["adjp"]))
    arcs = set(zip(src.tolist(), g["adjncy"].tolist()))
    for u in range(n):
        if m[u] != u:
            assert (u, int(m[u])) in arcs, f"matched along a non-edge {u}-{m[u]}"
    if maximal:
        single = m == np.arange(n)
        bad = single[src] & single[g["adjncy"]]
        assert not np.any(bad), "not maximal: an edge joins two unmatched vertices"


def check_level(g: Dict, match: np.ndarray, cmap: np.ndarray, n_c: int, coarse: Dict) -> None:
    """Per-level invariants of DESIGN.md §2.4 (north_star's list)."""
    g = np_graph(g)
    c = np_graph(coarse)
    n = g["n"]
    m = np.asarray(match, dtype=np.int64)
    cm = np.asarray(cmap, dtype=np.int64)
    pairs = int(np.sum(m > np.arange(n)))
    assert n_c == n - pairs
    # CM onto [0, n_c), increasing over leaders, partners share the leader's id
    lead = np.arange(n) <= m
    assert np.array_equal(cm[lead], np.arange(n_c))
    assert np.all(cm == cm[m])
    check_csr(c, "coarse")
    assert c["n"] == n_c
    assert int(c["vwgt"].sum()) == int(g["vwgt"].sum())
    src = np.repeat(np.arange(n), np.diff(g["adjp"]))
    collapsed = int(g["adjwgt"][m[src] == g["adjncy"]].sum())      # both arc directions
    assert int(c["adjwgt"].sum()) == int(g["adjwgt"].sum()) - collapsed
    adj = c["adjncy"]
    if len(adj) > 1:
        rows = np.repeat(np.arange(n_c), np.diff(c["adjp"]))
        same_row = rows[1:] == rows[:-1]
        assert np.all(np.diff(adj)[same_row] > 0), "coarse row not strictly increasing"


def contract_by_sparse_triple_product(g: Dict, cmap: np.ndarray, n_c: int) -> Dict:
    """Coarse graph as the off-diagonal of P^T A P and P^T vwgt (scipy.sparse), with P the
    0/1 fine->coarse assignment matrix: an independent formulation of P12.s26-28."""
    import scipy.sparse as sp
    g = np_graph(g)
    n = g["n"]
    A = sp.csr_matrix((g["adjwgt"], g["adjncy"], g["adjp"]), shape=(n, n))
    P = sp.csr_matrix((np.ones(n, dtype=np.int64), (np.arange(n), np.asarray(cmap))), shape=(n, n_c))
    C = (P.T @ A @ P).tocsr()
    C.setdiag(0)
    C.eliminate_zeros()
    C.sort_indices()
    return {"adjp": C.indptr.astype(np.int64), "adjncy": C.indices.astype(np.int64),
            "adjwgt": C.data.astype(np.int64),
            "vwgt": np.asarray(P.T @ g["vwgt"]).astype(np.int64).ravel()}
