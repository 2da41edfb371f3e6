"""Coarse-level tail (csrc/small.cu), -m gpu: once a level's graph fits one
SM's shared memory, one CTA runs every remaining level in one launch.  Its hierarchies must be
bit-identical to the oracle and to the level kernels (GP_SMALL=0 forces the level kernels)."""
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


def _run(gp, ctx, g, small, **kw):
    old = os.environ.get("GP_SMALL")
    os.environ["GP_SMALL"] = "1" if small else "0"
    try:
        l0 = ctx.launch_count()
        got = gpu_coarsen(gp, ctx, g, **kw)
        return got, ctx.launch_count() - l0
    finally:
        if old is None:
            del os.environ["GP_SMALL"]
        else:
            os.environ["GP_SMALL"] = old


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
    small, l_small = _run(gp, ctx, g, True, **kw)
    big, l_big = _run(gp, ctx, g, False, **kw)
    assert_levels_equal(small, ref, f"{name} tail")
    assert_levels_equal(big, ref, f"{name} level kernels")
    if len(ref) > 1:
        assert l_small < l_big, (l_small, l_big)  # the tail really ran (fewer launches)


def test_tail_is_one_launch_on_c1(gp, ctx):
    g = G.make_config("C1")
    got, launches = _run(gp, ctx, g, True, threshold=100)
    assert len(got) == 6 and launches <= 2  # (+ the input's size record copy is not a launch)
