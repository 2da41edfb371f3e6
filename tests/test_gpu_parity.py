"""GPU parity (-m gpu): the CUDA path through the C ABI equals the oracle bit for bit.

Sizes span several tiles of every kernel and a ragged tail; the full-size configs run in
the launch configuration bench.py times.  Edge cases: empty and isolated graphs, hub rows
that take the CTA proposal bin and every contraction bin, unit-weight wavefronts, the
max_rounds cap, invalid inputs and weight overflow.
"""
import json
import os

import numpy as np
import pytest
import torch

import graphgen as G
import oracle
from checks import check_level, check_matching
from gpu_helpers import assert_levels_equal, gpu_coarsen, to_device

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


@pytest.fixture(scope="module")
def gp():
    import paper_conf_ipps_goodarzibg16_b200.gp as gp
    return gp


@pytest.fixture(scope="module")
def ctx(gp):
    c = gp.Context(0)
    yield c
    c.close()


def _golden():
    with open(os.path.join(GOLDEN, "hand_worked.json")) as f:
        return json.load(f)["cases"]


@pytest.mark.parametrize("case", _golden(), ids=lambda c: c["name"])
def test_golden_level(gp, ctx, case):
    g = G.from_edge_list(case["n"], case["edges"])
    d = to_device(g)
    Gr = gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"], validate=True)
    m = torch.empty(case["n"], dtype=torch.int32, device="cuda")
    rounds = Gr.match_level(m)
    assert rounds == case["rounds"]
    assert m.cpu().tolist() == case["match"]
    cm = torch.empty_like(m)
    C = Gr.contract_level(m, cm)
    assert cm.cpu().tolist() == case["cmap"]
    c = C.download()
    assert c["n"] == case["n_coarse"]
    for k in ("adjp", "adjncy", "adjwgt", "vwgt"):
        assert c[k].tolist() == case["coarse"][k], k


def _random_cases():
    out = []
    for seed in range(24):
        n = [1, 2, 7, 100, 1000, 5000, 20000, 70001][seed % 8]
        m = n * [1, 2, 4, 8][seed % 4]
        wmax = [1, 2, 5, 100][(seed // 2) % 4]
        out.append((n, m, seed, wmax))
    return out


@pytest.mark.parametrize("n,m,seed,wmax", _random_cases())
def test_random_graphs_all_levels(gp, ctx, n, m, seed, wmax):
    g = G.random_graph(n, m, seed, wmax)
    ref = oracle.coarsen_to(g, threshold=8)
    got = gpu_coarsen(gp, ctx, g, threshold=8)
    assert_levels_equal(got, ref, f"er{n}_{m}_{seed}_{wmax}")


SMALL = {
    "C1": lambda: G.make_config("C1"),
    "C2_2^16": lambda: G.rgg(1 << 16),
    "C3_256": lambda: G.delaunay_like(256),
    "C3_300": lambda: G.delaunay_like(300),
    "C4_s14": lambda: G.rmat(14),
    # weights [1,4] as C4: 785 rows > 1024 arcs (multi-CTA hub phase), 18 > 4096, max 15.8 K
    # (C1h long rows: smem-sorted runs + merge-path merges + windowed run sums)
    "C4_s17_w4": lambda: G.rmat(17, wmax=4),
    "C4_s12_unit": lambda: G.rmat(12, unit=True),
    "C5_256": lambda: G.road_like(256),
    "grid_unit_128": lambda: G.grid2d(128, 128),
}


@pytest.mark.parametrize("name", list(SMALL))
def test_small_configs_all_levels(gp, ctx, name):
    g = SMALL[name]()
    ref = oracle.coarsen_to(g, threshold=100)
    got = gpu_coarsen(gp, ctx, g, threshold=100)
    assert_levels_equal(got, ref, name)
    cur = g
    for lvl in got:
        check_matching(cur, lvl["match"], maximal=True)
        check_level(cur, lvl["match"], lvl["cmap"], lvl["n_coarse"], lvl["coarse"])
        cur = lvl["coarse"]


def _star(n_leaves, wmax=100, extra_ring=True):
    edges = [(0, i, 1 + (i * 37) % wmax) for i in range(1, n_leaves + 1)]
    if extra_ring:
        edges += [(i, i + 1, 1 + (i * 11) % wmax) for i in range(1, n_leaves)]
    return G.from_edge_list(n_leaves + 1, edges)


@pytest.mark.parametrize("leaves", [40, 300, 5000, 9000, 20000])
def test_hub_rows_every_bin(gp, ctx, leaves):
    # a hub of degree `leaves` takes the warp / CTA proposal bins and, after contraction,
    # the warp / CTA / global merge bins
    g = _star(leaves)
    ref = oracle.coarsen_to(g, threshold=2)
    got = gpu_coarsen(gp, ctx, g, threshold=2)
    assert_levels_equal(got, ref, f"star{leaves}")


def test_two_hubs_shared_neighbourhood(gp, ctx):
    # two hubs matched together whose rows overlap: a long merged row with many duplicates
    k = 12000
    edges = [(0, 1, 1000)] + [(0, i, 1 + i % 50) for i in range(2, k)] + [(1, i, 1 + i % 70) for i in range(2, k)]
    edges += [(i, i + 1, 1 + i % 3) for i in range(2, k - 1)]
    g = G.from_edge_list(k, edges)
    assert_levels_equal(gpu_coarsen(gp, ctx, g, threshold=2), oracle.coarsen_to(g, threshold=2), "twohubs")


def test_empty_and_isolated(gp, ctx):
    for n in (0, 1, 5, 3000):
        g = G.from_edge_list(n, [])
        ref = oracle.coarsen_to(g, threshold=0)
        got = gpu_coarsen(gp, ctx, g, threshold=0)
        assert_levels_equal(got, ref, f"isolated{n}")


def test_single_edge_and_ragged_tail(gp, ctx):
    for n in (2, 2047, 2048, 2049, 4097):
        g = G.from_edge_list(n, [(n - 2, n - 1, 3)] if n >= 2 else [])
        assert_levels_equal(gpu_coarsen(gp, ctx, g, threshold=0), oracle.coarsen_to(g, threshold=0), f"edge{n}")


@pytest.mark.parametrize("cap", [1, 2, 5])
def test_max_rounds_cap(gp, ctx, cap):
    g = G.grid2d(40, 40)
    ref = oracle.coarsen_to(g, threshold=100, max_rounds=cap)
    got = gpu_coarsen(gp, ctx, g, threshold=100, max_rounds=cap)
    assert_levels_equal(got, ref, f"cap{cap}")


def test_deterministic_and_host_input(gp, ctx):
    g = G.rmat(13)
    a = gpu_coarsen(gp, ctx, g, threshold=100)
    b = gpu_coarsen(gp, ctx, g, threshold=100)
    assert_levels_equal(a, b, "repeat")
    # host (pinned) input path of gp_graph_create gives the same graph
    h = {k: g[k].contiguous().pin_memory() for k in ("adjp", "adjncy", "adjwgt", "vwgt")}
    Gh = gp.Graph.create(ctx, h["adjp"], h["adjncy"], h["adjwgt"], h["vwgt"])
    back = Gh.download()
    for k in ("adjp", "adjncy", "adjwgt", "vwgt"):
        assert torch.equal(back[k], g[k].cpu())


def test_null_weights_mean_unit(gp, ctx):
    g = G.grid2d(20, 20)
    d = to_device(g)
    Gr = gp.Graph.create(ctx, d["adjp"], d["adjncy"], None, None)
    back = Gr.download()
    assert set(back["adjwgt"].tolist()) == {1} and set(back["vwgt"].tolist()) == {1}


def test_validate_rejects_bad_graphs(gp, ctx):
    good = G.grid2d(6, 6)
    d = to_device(good)
    gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"], validate=True)
    bad_cases = {}
    x = {k: v.clone() for k, v in good.items() if isinstance(v, torch.Tensor)}
    x["adjncy"][3] = 999
    bad_cases["range"] = x
    x = {k: v.clone() for k, v in good.items() if isinstance(v, torch.Tensor)}
    x["adjwgt"][5] = 7
    bad_cases["asymmetric"] = x
    x = {k: v.clone() for k, v in good.items() if isinstance(v, torch.Tensor)}
    x["adjncy"][0] = 0
    bad_cases["selfloop"] = x
    x = {k: v.clone() for k, v in good.items() if isinstance(v, torch.Tensor)}
    x["adjwgt"][0] = 0
    bad_cases["weight"] = x
    for name, b in bad_cases.items():
        db = to_device(b)
        with pytest.raises(gp.GPError) as e:
            gp.Graph.create(ctx, db["adjp"], db["adjncy"], db["adjwgt"], db["vwgt"], validate=True)
        assert e.value.status == 2, name


def test_weight_overflow_rejected(gp, ctx):
    g = G.from_edge_list(3, [(0, 1, 2**30), (1, 2, 2**30)])
    d = to_device(g)
    with pytest.raises(gp.GPError) as e:
        gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"])
    assert e.value.status == 3


# ---- stop-rule boundaries (R12 / R13), the same cases as the oracle pins ---------------------
def test_stop_rule_boundaries(gp, ctx):
    g = G.make_config("C1")
    for thr in (64, 63, 4096):
        assert_levels_equal(gpu_coarsen(gp, ctx, g, threshold=thr), oracle.coarsen_to(g, threshold=thr), f"C1 thr{thr}")
    got = gpu_coarsen(gp, ctx, g, threshold=64)
    assert len(got) == 6 and got[-1]["n_coarse"] == 64
    for n in (20, 21):
        g = G.from_edge_list(n, [(3, 11, 5)])
        ref = oracle.coarsen_to(g, threshold=1)
        got = gpu_coarsen(gp, ctx, g, threshold=1)
        assert len(got) == (2 if n == 20 else 1)
        assert_levels_equal(got, ref, f"one-edge{n}")
    g = G.from_edge_list(20, [(3, 11, 5)])
    assert_levels_equal(gpu_coarsen(gp, ctx, g, threshold=1, stall_ratio_pct=94),
                        oracle.coarsen_to(g, threshold=1, stall_ratio_pct=94), "stall94")
    g = G.make_config("C1")
    for ml in (3, 6):
        assert_levels_equal(gpu_coarsen(gp, ctx, g, threshold=100, max_levels=ml),
                            oracle.coarsen_to(g, threshold=100, max_levels=ml), f"maxlev{ml}")


# ---- unsorted rows and non-unit vertex weights (input contract R15: any neighbour order) ----
# Every other GPU parity input has rows sorted by neighbour id and unit level-0 vertex weights;
# these run the same kernels on seeded per-row shuffles with vwgt = 1 + u % 7, validated.
SHUFFLED = {
    "C3_256": lambda: G.delaunay_like(256),
    "C4_s14": lambda: G.rmat(14),
    "C4_s17_w4": lambda: G.rmat(17, wmax=4),
    "C5_256": lambda: G.road_like(256),
    "C2_2^14": lambda: G.rgg(1 << 14),
    "star5000": lambda: _star(5000),
    "star20000": lambda: _star(20000),
}


@pytest.mark.parametrize("name", list(SHUFFLED))
@pytest.mark.parametrize("seed", [1, 2])
def test_shuffled_rows_varied_vwgt(gp, ctx, name, seed):
    g = G.varied_vwgt(G.shuffle_rows(SHUFFLED[name](), seed))
    thr = 2 if name.startswith("star") else 100
    ref = oracle.coarsen_to(g, threshold=thr)
    got = gpu_coarsen(gp, ctx, g, threshold=thr, validate=True)
    assert_levels_equal(got, ref, f"{name}_shuf{seed}")
    # the coarse vertex weights really are the non-unit sums
    assert got[0]["coarse"]["vwgt"].max() > 2


def test_validate_unsorted_rows(gp, ctx):
    """GP_VALIDATE on unsorted rows: an exact per-row hash check (duplicates, symmetry with
    equal weights), including a duplicate that is non-adjacent in its row and mirrored on the
    other side (order-independent fingerprints cannot see it)."""
    good = G.shuffle_rows(G.grid2d(6, 6, unit=False), 5)
    d = to_device(good)
    gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"], validate=True)
    # mirrored non-adjacent duplicate: row 0 = [1, 6] -> [1, 6, 1]? keep nnz: replace arcs so that
    # vertex 7 lists 8 twice (non-adjacent) and vertex 8 lists 7 twice, weights equal
    n = 36
    edges = [(u, v, w) for u, v, w in [(i, j, 1 + (i * 7 + j) % 5) for i in range(n) for j in range(i + 1, n)
                                       if (j == i + 1 and (i + 1) % 6) or j == i + 6]]
    rows = {u: [] for u in range(n)}
    for u, v, w in edges:
        rows[u].append((v, w))
        rows[v].append((u, w))
    w78 = [w for v, w in rows[7] if v == 8][0]
    rows[7] = [(8, w78)] + [x for x in rows[7] if x[0] != 8] + [(8, w78)]
    rows[8] = [(7, w78)] + [x for x in rows[8] if x[0] != 7] + [(7, w78)]
    adjp = np.cumsum([0] + [len(rows[u]) for u in range(n)])
    adjncy = np.array([v for u in range(n) for v, _ in rows[u]], dtype=np.int32)
    adjwgt = np.array([w for u in range(n) for _, w in rows[u]], dtype=np.int32)
    bad = {"adjp": torch.tensor(adjp, dtype=torch.int32), "adjncy": torch.tensor(adjncy),
           "adjwgt": torch.tensor(adjwgt), "vwgt": torch.ones(n, dtype=torch.int32)}
    db = to_device(bad)
    with pytest.raises(gp.GPError) as e:
        gp.Graph.create(ctx, db["adjp"], db["adjncy"], db["adjwgt"], db["vwgt"], validate=True)
    assert e.value.status == 2 and "duplicate" in str(e.value)
    # unsorted and asymmetric weight
    x = {k: v.clone() for k, v in good.items() if isinstance(v, torch.Tensor)}
    x["adjwgt"][4] += 1
    dx = to_device(x)
    with pytest.raises(gp.GPError) as e:
        gp.Graph.create(ctx, dx["adjp"], dx["adjncy"], dx["adjwgt"], dx["vwgt"], validate=True)
    assert e.value.status == 2 and "asymmetric" in str(e.value)
    # unsorted and a missing reverse arc (arc retargeted)
    x = {k: v.clone() for k, v in good.items() if isinstance(v, torch.Tensor)}
    row0 = x["adjncy"][int(x["adjp"][0]):int(x["adjp"][1])].tolist()
    x["adjncy"][0] = [v for v in range(2, n) if v not in row0][0]
    dx = to_device(x)
    with pytest.raises(gp.GPError) as e:
        gp.Graph.create(ctx, dx["adjp"], dx["adjncy"], dx["adjwgt"], dx["vwgt"], validate=True)
    assert e.value.status == 2


# ---- gp_match_level + gp_contract_level called standalone on hub rows ------------------------
@pytest.mark.parametrize("name", ["C4_s17_w4", "star20000"])
def test_standalone_match_contract_levels(gp, ctx, name):
    """The two per-level entry points chained by the caller (not through gp_coarsen_to) on
    graphs whose rows take the hub proposal phase and the C1h merge bins."""
    g = {"C4_s17_w4": lambda: G.rmat(17, wmax=4), "star20000": lambda: _star(20000)}[name]()
    ref = oracle.coarsen_to(g, threshold=2)
    d = to_device(g)
    cur = gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"], validate=True)
    keep = []
    for i, lvl in enumerate(ref):
        n = cur.n
        assert n == lvl["n"]
        m = torch.empty(n, dtype=torch.int32, device="cuda")
        rounds = cur.match_level(m)
        assert rounds == lvl["rounds"], (i, rounds, lvl["rounds"])
        assert np.array_equal(m.cpu().numpy(), lvl["match"]), f"level {i}: match"
        cm = torch.empty_like(m)
        nxt = cur.contract_level(m, cm)
        assert np.array_equal(cm.cpu().numpy(), lvl["cmap"]), f"level {i}: cmap"
        c = nxt.download()
        for k in ("adjp", "adjncy", "adjwgt", "vwgt"):
            assert np.array_equal(c[k].numpy(), lvl["coarse"][k]), f"level {i}: coarse {k}"
        keep.append(cur)
        cur = nxt
    for x in keep + [cur]:
        x.close()


# ---- the paper's one-shot HEM + conflict self-match -------------------
@pytest.mark.parametrize("name", ["C3_256", "C5_256", "C4_s14", "C2_2^16"])
def test_one_shot_mode(gp, ctx, name):
    """max_rounds = 1 on the GPU is the paper's single HEM pass + conflict kernel (P18.s7-13)
    with the races removed: compared with checks.one_shot_hem (computed from the definition)
    at every level and with the oracle's capped hierarchy."""
    from checks import one_shot_hem
    g = SMALL[name]()
    got = gpu_coarsen(gp, ctx, g, threshold=100, max_rounds=1)
    assert_levels_equal(got, oracle.coarsen_to(g, threshold=100, max_rounds=1), f"{name} one-shot")
    cur = g
    for lvl in got:
        assert np.array_equal(lvl["match"].astype(np.int64), one_shot_hem(cur))
        cur = lvl["coarse"]
