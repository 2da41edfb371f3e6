"""ABI behaviour on the GPU (-m gpu): the NCCL transport with a 1-rank communicator, the
user allocator hook, the global weight-total check of the sharded create, handle lifetimes
in the binding, and the caller's current device being left alone."""
import numpy as np
import pytest
import torch

import graphgen as G
import oracle
from gpu_helpers import assert_levels_equal, gpu_coarsen, to_device

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gp():
    import paper_conf_ipps_goodarzibg16_b200.gp as gp
    return gp


def _levels(gp, H):
    out = []
    for i, info in enumerate(H.levels()):
        m, c = H.download_level(i)
        coarse = H.download_coarse(i)
        out.append({"n": info.n, "nnz": info.nnz, "n_coarse": info.n_coarse, "rounds": info.rounds,
                    "maximal": info.maximal, "stop_reason": info.stop_reason, "match": m.numpy(),
                    "cmap": c.numpy(), "coarse": {k: coarse[k].numpy() for k in ("adjp", "adjncy", "adjwgt", "vwgt")}})
    return out


@pytest.mark.parametrize("fold", ["off", "default"])
def test_nccl_transport_one_rank(gp, fold, monkeypatch):
    """gp_ctx_create_dist with a real (1-rank) NCCL communicator: gp_graph_create_dist, the
    sharded driver's ncclAllGather / grouped send-recv calls, bit-exact vs the oracle; with
    folding on, the gather of the coarse graph is an ncclAllGather too."""
    if fold == "off":
        monkeypatch.setenv("GP_FOLD_N", "0")
    else:
        monkeypatch.delenv("GP_FOLD_N", raising=False)
    uid = gp.nccl_unique_id()
    ctx = gp.Context(0, nccl_id=uid, rank=0, nranks=1)
    assert ctx.dist_info() == (0, 1)
    g = G.delaunay_like(96)
    d = to_device(g)
    Gr = gp.Graph.create_dist(ctx, g["n"], 0, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"])
    H = Gr.coarsen_to(100)
    assert_levels_equal(_levels(gp, H), oracle.coarsen_to(g, threshold=100), "nccl1")
    H.close()
    Gr.close()
    # global weight totals are checked on every rank (R14): this shard alone overflows
    bad = G.from_edge_list(3, [(0, 1, 2**30), (1, 2, 2**30)])
    db = to_device(bad)
    with pytest.raises(gp.GPError) as e:
        gp.Graph.create_dist(ctx, 3, 0, db["adjp"], db["adjncy"], db["adjwgt"], db["vwgt"])
    assert e.value.status == 3
    # shards must tile [0, n_global)
    with pytest.raises(gp.GPError) as e:
        gp.Graph.create_dist(ctx, g["n"] + 5, 0, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"])
    assert e.value.status == 1
    ctx.close()


def test_torch_allocator_hook(gp):
    """gp_ctx_set_allocator routed to torch's caching allocator: same results; switching is
    refused while graphs / hierarchies hold buffers of the current allocator."""
    ctx = gp.Context(0)
    ctx.use_torch_allocator()
    before = torch.cuda.memory_allocated()
    g = G.rmat(13)
    d = to_device(g)
    Gr = gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"])
    assert torch.cuda.memory_allocated() > before  # the graph lives in torch's pool
    H = Gr.coarsen_to(100)
    assert_levels_equal(_levels(gp, H), oracle.coarsen_to(g, threshold=100), "torch-alloc")
    with pytest.raises(gp.GPError) as e:
        ctx.set_allocator(None, None)
    assert e.value.status == 1 and "still hold" in str(e.value)
    H.close()
    Gr.close()
    ctx.set_allocator(None, None)  # nothing alive any more: back to cudaMallocAsync
    got = gpu_coarsen(gp, ctx, g, threshold=100)
    assert_levels_equal(got, oracle.coarsen_to(g, threshold=100), "default-alloc")
    ctx.close()


def test_binding_lifetimes(gp):
    ctx = gp.Context(0)
    g = G.grid2d(16, 16)
    d = to_device(g)
    Gr = gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"])
    coarse = Gr.coarsen_to(10).level(0).coarse   # the hierarchy object is only referenced by `coarse`
    assert coarse.download()["n"] == 128         # ... and stays alive through it
    H = Gr.coarsen_to(10)
    c0 = H.level(0).coarse
    H.close()
    with pytest.raises(RuntimeError):
        c0.download()                            # borrowed from a closed hierarchy
    H2 = Gr.coarsen_to(10)
    ctx.close()                                  # closes H2 and Gr first
    assert H2.handle is None and Gr.handle is None
    with pytest.raises(RuntimeError):
        len(H2)
    with pytest.raises(RuntimeError):
        Gr.download()


def test_current_device_is_restored(gp):
    dev = torch.cuda.current_device()
    ctx = gp.Context(0)
    g = G.grid2d(8, 8)
    got = gpu_coarsen(gp, ctx, g, threshold=4)
    assert torch.cuda.current_device() == dev
    assert_levels_equal(got, oracle.coarsen_to(g, threshold=4), "grid8")
    ctx.close()
