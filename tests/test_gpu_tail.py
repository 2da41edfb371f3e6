"""Coarse-level tail, -m gpu: once the level bounds are small, ONE launch runs
every remaining level -- one CTA with the graph in shared memory (csrc/small.cu) when it fits one
SM, else every SM with its vertex range and rows in shared memory (csrc/part.cu), or (opt-in)
one thread-block cluster with the graph in L2 (csrc/medium.cu).  Each hierarchy must be
bit-identical to the oracle and to the level kernels, in every mode:
  small    (default)                  single CTA when it fits, else the partitioned grid tail
                                      when it fits, else the level kernels
  part     (GP_SMALL=0)               the partitioned grid tail even for graphs that fit one SM
  part_many (GP_SMALL=0, GP_PART_W=256)  ... on many CTAs (ranges of a few vertices: most pairs
                                      and arcs cross CTA ranges)
  part_global (+ GP_PART_GARCS=1, GP_PART_WCAP=64)  rows and most window lookups read from
                                      global memory (the paths of graphs that do not fit)
  part_gstage (GP_SMALL=0, GP_PART_GSTAGE=1)  merged rows staged in global memory (levels whose
                                      merged rows do not fit shared memory) instead of shared
  medium   (GP_SMALL=0, GP_MEDIUM=1)  the cluster kernel (opt-in: measured slower)
  levels   (GP_SMALL=0, GP_MEDIUM=0, GP_PART=0)  the grid-wide level kernels only."""
import os

import numpy as np
import pytest

import graphgen as G
import oracle
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


MODES = {
    "small": {},
    "part": {"GP_SMALL": "0"},
    "part_many": {"GP_SMALL": "0", "GP_PART_W": "256"},
    "part_global": {"GP_SMALL": "0", "GP_PART_W": "256", "GP_PART_GARCS": "1", "GP_PART_WCAP": "64"},
    "part_gstage": {"GP_SMALL": "0", "GP_PART_GSTAGE": "1"},
    "medium": {"GP_SMALL": "0", "GP_MEDIUM": "1"},
    "levels": {"GP_SMALL": "0", "GP_MEDIUM": "0", "GP_PART": "0"},
}
KNOBS = ("GP_SMALL", "GP_MEDIUM", "GP_PART", "GP_PART_W", "GP_PART_GARCS", "GP_PART_WCAP", "GP_PART_GSTAGE")


def _run(gp, ctx, g, mode, **kw):
    env = MODES[mode]
    old = {k: os.environ.get(k) for k in KNOBS}
    for k in old:
        os.environ.pop(k, None)
    os.environ.update(env)
    try:
        l0 = ctx.launch_count()
        got = gpu_coarsen(gp, ctx, g, **kw)
        return got, ctx.launch_count() - l0
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


def _star(n_leaves, wmax=100):
    edges = [(0, i, 1 + (i * 37) % wmax) for i in range(1, n_leaves + 1)]
    edges += [(i, i + 1, 1 + (i * 11) % wmax) for i in range(1, n_leaves)]
    return G.from_edge_list(n_leaves + 1, edges)


CASES = {
    "C1": (lambda: G.make_config("C1"), dict(threshold=100)),
    "C1_thr64": (lambda: G.make_config("C1"), dict(threshold=64)),
    "C1_rm": (lambda: G.make_config("C1"), dict(threshold=100, tie_seed=0x9E3779B9)),
    "C1_cap2": (lambda: G.make_config("C1"), dict(threshold=100, max_rounds=2)),
    "C1_maxlev3": (lambda: G.make_config("C1"), dict(threshold=100, max_levels=3)),
    "grid_unit_40": (lambda: G.grid2d(40, 40), dict(threshold=10)),
    "delaunay_40": (lambda: G.delaunay_like(40), dict(threshold=10)),
    "rmat10_shuf_vw": (lambda: G.varied_vwgt(G.shuffle_rows(G.rmat(10), 3)), dict(threshold=10)),
    "star1500": (lambda: _star(1500), dict(threshold=2)),
    "star5000": (lambda: _star(5000), dict(threshold=2)),  # a merged row > 2048 keys (global staging)
    "road_48": (lambda: G.road_like(48), dict(threshold=5)),
    "isolated": (lambda: G.from_edge_list(300, []), dict(threshold=0)),
    "one_edge20": (lambda: G.from_edge_list(20, [(3, 11, 5)]), dict(threshold=1)),
    # starts on the level kernels and enters the tail when the bounds fit
    "C3_128": (lambda: G.delaunay_like(128), dict(threshold=100)),
    "C2_2^14": (lambda: G.rgg(1 << 14), dict(threshold=100)),
}


@pytest.mark.parametrize("name", list(CASES))
def test_tail_equals_oracle_and_level_kernels(gp, ctx, name):
    make, kw = CASES[name]
    g = make()
    ref = oracle.coarsen_to(g, **kw)
    launches = {}
    for mode in MODES:
        got, launches[mode] = _run(gp, ctx, g, mode, **kw)
        assert_levels_equal(got, ref, f"{name} {mode}")
    if len(ref) > 1:  # the tail really ran (fewer launches than the level kernels)
        assert launches["medium"] < launches["levels"], launches
        assert launches["part"] < launches["levels"], launches
        if g["n"] <= 8192:
            assert launches["small"] < launches["levels"], launches


def test_tail_is_one_launch_on_c1(gp, ctx):
    g = G.make_config("C1")
    got, launches = _run(gp, ctx, g, "small", threshold=100)
    assert len(got) == 6 and launches <= 2  # (graph creation's totals kernel + the tail)


@pytest.mark.parametrize("name", ["C3_512", "C2_2^16", "road_256", "rmat14_w4"])
def test_medium_tail_mid_hierarchy(gp, ctx, name):
    """Graphs whose hierarchies enter the grid / cluster tail after a few level kernels."""
    g = {"C3_512": lambda: G.delaunay_like(512), "C2_2^16": lambda: G.rgg(1 << 16),
         "road_256": lambda: G.road_like(256), "rmat14_w4": lambda: G.rmat(14, wmax=4)}[name]()
    ref = oracle.coarsen_to(g, threshold=100)
    for mode in ("small", "part_many", "part_global", "medium", "levels"):
        got, _ = _run(gp, ctx, g, mode, threshold=100)
        assert_levels_equal(got, ref, f"{name} {mode}")


@pytest.mark.parametrize("name", ["C3_512", "rgg_2^16", "road_256", "grid_shuf_vw"])
def test_windowed_match_opt_in(gp, ctx, name):
    """The opt-in windowed big-level matching (csrc/match_win.cu, GP_WIN=1), forced onto small
    levels (GP_WIN_N), with and without the grid tail: bit-identical to the oracle."""
    g = {"C3_512": lambda: G.delaunay_like(512), "rgg_2^16": lambda: G.rgg(1 << 16),
         "road_256": lambda: G.road_like(256),
         "grid_shuf_vw": lambda: G.varied_vwgt(G.shuffle_rows(G.grid2d(200, 200), 5))}[name]()
    ref = oracle.coarsen_to(g, threshold=100)
    old = {k: os.environ.get(k) for k in ("GP_WIN", "GP_WIN_N", "GP_PART")}
    try:
        os.environ["GP_WIN"] = "1"
        os.environ["GP_WIN_N"] = "2000"
        for part in ("1", "0"):
            os.environ["GP_PART"] = part
            got = gpu_coarsen(gp, ctx, g, threshold=100)
            assert_levels_equal(got, ref, f"{name} windowed part={part}")
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


@pytest.mark.parametrize("mode", ["small", "part", "part_many"])
@pytest.mark.parametrize("name", ["C1", "C3_128", "star1500"])
def test_tail_continues_across_launches(gp, ctx, name, mode):
    """A tail launch holds at most GP_TAIL_SLOTS levels (default 12); a deeper hierarchy
    continues with further launches from the last tail level's output.  With 2 slots every
    hierarchy here needs several launches: still bit-identical to the oracle."""
    make, kw = CASES[name]
    g = make()
    ref = oracle.coarsen_to(g, **kw)
    old = os.environ.get("GP_TAIL_SLOTS")
    os.environ["GP_TAIL_SLOTS"] = "2"
    try:
        got, launches = _run(gp, ctx, g, mode, **kw)
        assert_levels_equal(got, ref, f"{name} {mode} 2 slots")
    finally:
        if old is None:
            os.environ.pop("GP_TAIL_SLOTS", None)
        else:
            os.environ["GP_TAIL_SLOTS"] = old
