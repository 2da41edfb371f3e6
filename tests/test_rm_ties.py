"""RM tie priority (reading R17 of DESIGN.md §2; P18.s8: "If all the edges have the same
weight, a random matching (RM) [14] method is used in an iterative fashion where each vertex
chooses one of its unmatched vertices randomly").

The random choice is made deterministic by a seeded priority h_s(v) = lowbias32(v ^ s):
among neighbours of equal edge weight, the lower h_s(v) wins (seed 0 = the north_star rule,
lower id).  Pins of the seeded oracle (-m "not gpu"), none of which re-calls its code:
  * an independent Python transcription of lowbias32 (the constants of include/gp.h) and its
    bijectivity on a sample (distinct priorities are what the termination lemma needs);
  * equality with the textbook sequential greedy matching under the edge order
    (w desc, min h asc, max h asc) -- the same theorem that pins the seed-0 rule (§2.2);
  * equality with the (separately pinned) seed-0 oracle on the graph relabeled by the rank
    of h_s, mapped back;
  * seed independence when all weights are distinct; maximality and the 1/2 bound by brute
    force; the unit-grid wavefront (C1: 95 rounds at level 0) is gone.
The -m gpu tests compare the CUDA path (gp_match_level_ex, gp_coarsen_to with tie_seed, the
sharded loopback path) with the seeded oracle element by element.
"""
import numpy as np
import pytest
import torch

import graphgen as G
import oracle
from checks import check_matching, edge_list, max_weight_matching_bruteforce

M32 = 0xFFFFFFFF
SEEDS = [1, 0x9E3779B9, 12345, M32]


def lowbias32(v: int, s: int) -> int:
    x = (v ^ s) & M32
    x ^= x >> 16
    x = (x * 0x7FEB352D) & M32
    x ^= x >> 15
    x = (x * 0x846CA68B) & M32
    x ^= x >> 16
    return x


def greedy_h(n, edges, s):
    """Sequential greedy matching, edges by (w desc, min h asc, max h asc)."""
    h = [lowbias32(v, s) for v in range(n)]
    m = np.full(n, -1, dtype=np.int64)
    for u, v, w in sorted(edges, key=lambda e: (-e[2], min(h[e[0]], h[e[1]]), max(h[e[0]], h[e[1]]))):
        if m[u] < 0 and m[v] < 0:
            m[u], m[v] = v, u
    for u in range(n):
        if m[u] < 0:
            m[u] = u
    return m


def test_tie_hash_transcription():
    rng = np.random.default_rng(5)
    for s in SEEDS + [0]:
        for v in [0, 1, 2, 3, 12345, 2**31 - 1] + rng.integers(0, 2**31, 200).tolist():
            assert oracle.tie_hash(v, s) == lowbias32(v, s)
    # bijective on a window: distinct priorities per row
    for s in SEEDS:
        assert len({lowbias32(v, s) for v in range(1 << 16)}) == 1 << 16


@pytest.mark.parametrize("seed", range(40))
def test_seeded_equals_greedy_h_order(seed):
    n = 5 + (seed * 11) % 70
    g = G.random_graph(n, n * (1 + seed % 4), seed + 900, wmax=[1, 2, 3, 100][seed % 4])
    s = SEEDS[seed % len(SEEDS)]
    m, _, maximal = oracle.match_level(g, tie_seed=s)
    assert maximal
    assert np.array_equal(m.astype(np.int64), greedy_h(n, edge_list(g), s))


@pytest.mark.parametrize("seed", range(10))
def test_seeded_equals_relabeled_default_rule(seed):
    g = G.random_graph(300, 1200, seed + 40, wmax=[1, 3][seed % 2])
    n = 300
    s = SEEDS[seed % len(SEEDS)]
    rank = np.argsort(np.argsort([lowbias32(v, s) for v in range(n)], kind="stable"), kind="stable")
    h = G.from_edge_list(n, [(int(rank[u]), int(rank[v]), w) for u, v, w in edge_list(g)])
    ms, rs, _ = oracle.match_level(g, tie_seed=s)
    mr, rr, _ = oracle.match_level(h)
    assert rs == rr
    assert np.array_equal(rank[ms], mr[rank])


def test_seed_irrelevant_with_distinct_weights():
    g = G.random_graph(200, 800, 77, wmax=1 << 30)
    ws = [w for _, _, w in edge_list(g)]
    if len(set(ws)) != len(ws):
        pytest.skip("weight collision")
    m0, r0, _ = oracle.match_level(g)
    for s in SEEDS:
        m, r, _ = oracle.match_level(g, tie_seed=s)
        assert r == r0 and np.array_equal(m, m0)


@pytest.mark.parametrize("seed", range(60))
def test_seeded_bruteforce_small(seed):
    n = 2 + seed % 9
    g = G.random_graph(n, 2 * n, seed + 700, wmax=[1, 3, 10][seed % 3])
    m, _, maximal = oracle.match_level(g, tie_seed=SEEDS[seed % len(SEEDS)])
    assert maximal
    check_matching(g, m, maximal=True)
    edges = edge_list(g)
    assert 2 * sum(w for u, v, w in edges if m[u] == v) >= max_weight_matching_bruteforce(n, edges)


def test_rm_breaks_unit_wavefront():
    # C1 (64x64 unit grid) takes 95 rounds at level 0 with the lower-id rule: ties follow the
    # row-major ids.  Hashed priorities are uncorrelated with the geometry.
    g = G.make_config("C1")
    base = oracle.coarsen_to(g, threshold=100)
    assert base[0]["rounds"] == 95
    for s in SEEDS:
        lv = oracle.coarsen_to(g, threshold=100, tie_seed=s)
        assert max(l["rounds"] for l in lv) < 30
        assert lv[-1]["coarse"]["vwgt"].sum() == 4096


def star(leaves: int, w: int = 1):
    return G.from_edge_list(leaves + 1, [(0, i, w) for i in range(1, leaves + 1)])


@pytest.mark.parametrize("s", SEEDS)
def test_seeded_star_closed_form(s):
    # every leaf proposes to the hub; the hub proposes to the leaf of lowest h_s, which is
    # its partner; every other leaf is then dead (its only neighbour is matched)
    n = 3001
    m, rounds, maximal = oracle.match_level(star(n - 1), tie_seed=s)
    best = min(range(1, n), key=lambda v: lowbias32(v, s))
    assert m[0] == best and m[best] == 0 and rounds == 1 and maximal
    assert all(m[v] == v for v in range(1, n) if v != best)


def test_seeded_max_rounds_cap():
    g = G.grid2d(16, 16)
    m, r, maximal = oracle.match_level(g, max_rounds=1, tie_seed=SEEDS[1])
    assert r == 1 and not maximal
    check_matching(g, m, maximal=False)


# ----------------------------------------------------------------------------- GPU parity

GPU_GRAPHS = {
    "C1": lambda: G.make_config("C1"),
    "grid96_unit": lambda: G.grid2d(96, 96, unit=True),
    "delaunay128_w3": lambda: G.delaunay_like(128, wmax=3),
    "rgg16k_unit": lambda: G.rgg(16384, wmax=1),
    "road128_w2": lambda: G.road_like(128, wmax=2),
    "rmat13_unit": lambda: G.rmat(13, 8, unit=True),
    "rmat14_w4": lambda: G.rmat(14, 16, wmax=4),
    "random_w1": lambda: G.random_graph(5000, 20000, seed=3, wmax=1),
    "star3000": lambda: star(3000),                      # hub row > 1024 arcs: hub phases
    "star50000": lambda: star(50000),                    # multi-CTA hub phase
    "isolated": lambda: G.from_edge_list(50, [(3, 7, 1), (7, 9, 1)]),
}


def _host(g):
    return {k: (v.cpu() if isinstance(v, torch.Tensor) else v) for k, v in g.items()}


@pytest.fixture(scope="module")
def gp():
    import paper_conf_ipps_goodarzibg16_b200.gp as gp
    return gp


@pytest.mark.gpu
@pytest.mark.parametrize("s", SEEDS[:2])
@pytest.mark.parametrize("name", list(GPU_GRAPHS))
def test_gpu_seeded_hierarchy_equals_oracle(gp, name, s):
    from gpu_helpers import assert_levels_equal, gpu_coarsen
    g = _host(GPU_GRAPHS[name]())
    ref = oracle.coarsen_to(g, threshold=20, tie_seed=s)
    got = gpu_coarsen(gp, gp.Context(0), g, threshold=20, tie_seed=s)
    assert_levels_equal(got, ref, f"{name} seed={s:#x}")


@pytest.mark.gpu
def test_gpu_match_level_ex(gp):
    from gpu_helpers import to_device
    g = _host(G.delaunay_like(96, wmax=2))
    d = to_device(g)
    ctx = gp.Context(0)
    Gr = gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"])
    for s in [0] + SEEDS:
        m = torch.empty(Gr.n, dtype=torch.int32, device="cuda")
        r = Gr.match_level(m, tie_seed=s)
        mo, ro, _ = oracle.match_level(g, tie_seed=s)
        assert r == ro and np.array_equal(m.cpu().numpy(), mo), f"seed {s:#x}"
    Gr.close()


@pytest.mark.gpu
@pytest.mark.parametrize("nranks", [2, 5])
@pytest.mark.parametrize("name", ["grid96_unit", "rmat13_unit", "road128_w2"])
def test_gpu_seeded_loopback_equals_oracle(gp, name, nranks):
    from gpu_helpers import assert_levels_equal, gpu_coarsen
    g = _host(GPU_GRAPHS[name]())
    ref = oracle.coarsen_to(g, threshold=20, tie_seed=SEEDS[1])
    got = gpu_coarsen(gp, gp.Context(0, loopback=nranks), g, threshold=20, tie_seed=SEEDS[1])
    assert_levels_equal(got, ref, f"{name} G={nranks}")


@pytest.mark.gpu
@pytest.mark.parametrize("name", ["grid96_unit", "rmat13_unit"])
def test_gpu_seeded_max_rounds_cap(gp, name):
    from gpu_helpers import assert_levels_equal, gpu_coarsen
    g = _host(GPU_GRAPHS[name]())
    ref = oracle.coarsen_to(g, threshold=20, max_rounds=2, tie_seed=SEEDS[2])
    got = gpu_coarsen(gp, gp.Context(0), g, threshold=20, max_rounds=2, tie_seed=SEEDS[2])
    assert_levels_equal(got, ref, f"{name} cap")
