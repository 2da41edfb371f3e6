"""Grid-wide merge of giant contraction rows (csrc/contract.cu phase_c1h_giant), -m gpu: rows
whose merged upper bound exceeds GP_GIANT_ROW (opt-in; measured slower on C4) are merged by every
CTA through a dense accumulator over the coarse ids instead of one CTA sorting them.  The
threshold is lowered here so that hub rows of small graphs take that path: every hierarchy must
stay bit-identical to the oracle (PAPER.md P20.s14-21 with R8-R10: summed, collapsed edge
dropped, sorted by coarse id)."""
import os

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


def _star(n_leaves, wmax=100):
    edges = [(0, i, 1 + (i * 37) % wmax) for i in range(1, n_leaves + 1)]
    edges += [(i, i + 1, 1 + (i * 11) % wmax) for i in range(1, n_leaves)]
    return G.from_edge_list(n_leaves + 1, edges)


CASES = {
    "rmat14": (lambda: G.rmat(14), 100, {}),
    "rmat17_w4": (lambda: G.rmat(17, wmax=4), 100, {}),
    "rmat14_shuf_vw": (lambda: G.varied_vwgt(G.shuffle_rows(G.rmat(14), 7)), 100, {}),
    "rmat14_rm": (lambda: G.rmat(14), 100, {"tie_seed": 0x9E3779B9}),
    "star20000": (lambda: _star(20000), 2, {}),
}


@pytest.mark.parametrize("giant", ["300", "2000"])
@pytest.mark.parametrize("name", list(CASES))
def test_giant_rows_equal_oracle(gp, ctx, name, giant):
    make, thr, kw = CASES[name]
    g = make()
    ref = oracle.coarsen_to(g, threshold=thr, **kw)
    old = {k: os.environ.get(k) for k in ("GP_GIANT_ROW", "GP_SMALL", "GP_PART")}
    try:
        os.environ["GP_GIANT_ROW"] = giant
        os.environ["GP_SMALL"] = "0"  # the level kernels (not the coarse-level tails) on every level
        os.environ["GP_PART"] = "0"
        got = gpu_coarsen(gp, ctx, g, threshold=thr, **kw)
        assert_levels_equal(got, ref, f"{name} giant>{giant}")
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
