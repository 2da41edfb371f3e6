"""The kernels' protocols, simulated on the CPU with adversarial in-phase
orders, reproduce the oracle exactly (-m "not gpu")."""
import numpy as np
import pytest

import graphgen as G
import oracle
from checks import np_graph
from protocol_sim import simulate_match


def _cases():
    out = []
    for seed in range(40):
        n = [5, 17, 60, 200][seed % 4]
        out.append((n, n * (1 + seed % 4), seed, [1, 2, 5, 100][(seed // 4) % 4]))
    return out


@pytest.mark.parametrize("n,m,seed,wmax", _cases())
def test_fused_round_protocol_equals_oracle(n, m, seed, wmax):
    g = G.random_graph(n, m, seed, wmax)
    gn = np_graph(g)
    ref_m, ref_r, ref_max = oracle.match_level(g)
    for order_seed in range(3):
        for cache in (True, False):
            sm, sr, smax = simulate_match(gn["adjp"], gn["adjncy"], gn["adjwgt"], seed=order_seed, use_cache=cache)
            assert np.array_equal(sm, ref_m) and sr == ref_r and smax == ref_max


@pytest.mark.parametrize("cap", [1, 2, 3])
def test_fused_round_protocol_cap(cap):
    g = G.grid2d(12, 12)
    gn = np_graph(g)
    ref_m, ref_r, ref_max = oracle.match_level(g, max_rounds=cap)
    sm, sr, smax = simulate_match(gn["adjp"], gn["adjncy"], gn["adjwgt"], seed=1, max_rounds=cap)
    assert np.array_equal(sm, ref_m) and sr == ref_r and smax == ref_max


def test_fused_round_protocol_meshes():
    for g in (G.delaunay_like(24), G.grid2d(10, 10), G.road_like(24), G.rmat(7)):
        gn = np_graph(g)
        ref_m, ref_r, ref_max = oracle.match_level(g)
        sm, sr, smax = simulate_match(gn["adjp"], gn["adjncy"], gn["adjwgt"], seed=5)
        assert np.array_equal(sm, ref_m) and sr == ref_r and smax == ref_max
