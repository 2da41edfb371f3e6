"""Generator checks (-m "not gpu"): hash stream, CSR validity, Table-I-like shapes."""
import numpy as np
import torch

import graphgen as G
from checks import check_csr, np_graph


def test_splitmix64_matches_scalar_reference():
    xs = [0, 1, 2, 3, 2**32, 2**63 - 1, 2**63, 2**64 - 1, 12345678901234567]
    t = torch.tensor([G._s64(x) for x in xs], dtype=torch.int64)
    got = [int(v) & G.MASK64 for v in G.splitmix64(t)]
    assert got == [G.splitmix64_int(x) for x in xs]
    # published first output of splitmix64 seeded with 0 (state += golden, then mix)
    assert G.splitmix64_int(0) == 0xE220A8397B1DCDAF


def test_weights_symmetric_and_in_range():
    u = torch.arange(1000, dtype=torch.int64)
    v = (u * 7919 + 13) % 1000
    a = G.edge_weights(u, v)
    b = G.edge_weights(v, u)
    assert torch.equal(a, b)
    assert int(a.min()) >= 1 and int(a.max()) <= 100


def test_c1_grid():
    g = G.make_config("C1")
    assert g["n"] == 4096 and g["nnz"] == 2 * 8064
    check_csr(g, "C1")
    assert set(np_graph(g)["adjwgt"].tolist()) == {1}


def test_delaunay_like_counts():
    side = 96
    g = G.delaunay_like(side)
    assert g["nnz"] // 2 == 2 * side * (side - 1) + (side - 1) ** 2
    check_csr(g, "C3-small")
    deg = np.diff(np_graph(g)["adjp"])
    assert deg.min() >= 2 and deg.max() <= 8


def test_rgg_degree_and_validity():
    g = G.rgg(1 << 12)
    check_csr(g, "C2-small")
    avg = g["nnz"] / g["n"]
    expect = np.pi * 0.55 ** 2 * np.log(1 << 12)
    assert abs(avg - expect) / expect < 0.1


def test_rmat_skew_and_validity():
    g = G.rmat(11)
    check_csr(g, "C4-small")
    deg = np.diff(np_graph(g)["adjp"])
    assert deg.max() > 20 * deg.mean()                  # skewed hubs
    assert (deg == 0).mean() > 0.05                     # isolated vertices exist


def test_road_like_degree():
    g = G.road_like(128)
    check_csr(g, "C5-small")
    assert abs(g["nnz"] / g["n"] - 2.5) < 0.1


def test_deterministic():
    a = G.rgg(1 << 11)
    b = G.rgg(1 << 11)
    for k in ("adjp", "adjncy", "adjwgt"):
        assert torch.equal(a[k], b[k])


def test_shuffle_rows_keeps_the_graph():
    g = G.rgg(1 << 10)
    s = G.shuffle_rows(g, 3)
    a, b = np_graph(g), np_graph(s)
    assert np.array_equal(a["adjp"], b["adjp"]) and np.array_equal(a["vwgt"], b["vwgt"])
    moved = 0
    for u in range(a["n"]):
        lo, hi = a["adjp"][u], a["adjp"][u + 1]
        x = sorted(zip(a["adjncy"][lo:hi], a["adjwgt"][lo:hi]))
        y = sorted(zip(b["adjncy"][lo:hi], b["adjwgt"][lo:hi]))
        assert x == y
        moved += int(not np.array_equal(a["adjncy"][lo:hi], b["adjncy"][lo:hi]))
    assert moved > a["n"] // 2      # most rows are really reordered
    check_csr(s, "shuffled")


def test_varied_vwgt():
    g = G.varied_vwgt(G.grid2d(5, 5), period=7)
    assert g["vwgt"].tolist() == [1 + u % 7 for u in range(25)]
