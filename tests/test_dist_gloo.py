"""The sharded protocol on the CPU: world_size 2 and 3 processes over gloo (127.0.0.1).

Each process runs tests/dist_protocol_sim.py -- the restatement of csrc/dist.cu's exchanges
(round all-gathers of boundary proposals with the P[P[v]] field, rank offsets of the coarse
ids, two-pass boundary CM resolution, partner rows sent to the leader's rank) -- on its
vertex range.  The gathered pieces must equal the oracle's hierarchy at every level: the
sharded run is the 1-GPU run.  The GPU path's parity at 2-8 ranks is
tests/test_gpu_dist.py (loopback transport); this file checks the protocol and the
process-group plumbing that bench.py --gpus N uses.
"""
import os
import socket
import sys
import traceback

import numpy as np
import pytest
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _graphs():
    import graphgen as G
    return {
        "grid12": G.grid2d(12, 12, unit=True),
        "delaunay16": G.delaunay_like(16),
        "road24": G.road_like(24),
        "rmat8": G.rmat(8, 8),
        "random": G.random_graph(300, 1200, seed=3),
    }


def _worker(rank, world, port, out_dir, threshold, max_rounds, tie_seed=0, fold_n=0):
    try:
        sys.path.insert(0, ROOT)
        sys.path.insert(0, os.path.join(ROOT, "tests"))
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        import torch.distributed as dist

        import dist_protocol_sim as sim

        dist.init_process_group("gloo", rank=rank, world_size=world)
        res = {}
        for name, g in _graphs().items():
            g = {k: (v.numpy() if hasattr(v, "numpy") else v) for k, v in g.items()}
            levels = sim.coarsen_to(sim.shard_of(g, rank, world), threshold, max_rounds=max_rounds,
                                    tie_seed=tie_seed, fold_n=fold_n)
            pieces = [None] * world
            dist.all_gather_object(pieces, [{"n": l["n"], "rounds": l["rounds"], "maximal": l["maximal"],
                                             "match": l["match"], "cmap": l["cmap"], "n_coarse": l["n_coarse"],
                                             "coarse": {"adjp": l["coarse"].adjp, "adjncy": l["coarse"].adjncy,
                                                        "adjwgt": l["coarse"].adjwgt, "vwgt": l["coarse"].vwgt}}
                                            for l in levels])
            res[name] = pieces
        if rank == 0:
            import pickle
            with open(os.path.join(out_dir, "result.pkl"), "wb") as f:
                pickle.dump(res, f)
        dist.barrier()
        dist.destroy_process_group()
    except Exception:
        with open(os.path.join(out_dir, f"error{rank}.txt"), "w") as f:
            f.write(traceback.format_exc())
        raise


def _concat(pieces, i):
    lv = [p[i] for p in pieces]
    adjp, adjncy, adjwgt, vwgt = [np.zeros(1, dtype=np.int64)], [], [], []
    off = 0
    for l in lv:
        c = l["coarse"]
        adjp.append(np.asarray(c["adjp"][1:]) + off)
        off += int(c["adjp"][-1])
        adjncy.append(c["adjncy"])
        adjwgt.append(c["adjwgt"])
        vwgt.append(c["vwgt"])
    return {"match": np.concatenate([l["match"] for l in lv]), "cmap": np.concatenate([l["cmap"] for l in lv]),
            "coarse": {"adjp": np.concatenate(adjp), "adjncy": np.concatenate(adjncy),
                       "adjwgt": np.concatenate(adjwgt), "vwgt": np.concatenate(vwgt)},
            "rounds": lv[0]["rounds"], "maximal": lv[0]["maximal"], "n_coarse": lv[0]["n_coarse"]}


@pytest.mark.parametrize("world,max_rounds,tie_seed,fold_n", [(2, 0, 0, 0), (3, 0, 0, 0), (2, 2, 0, 0),
                                                             (2, 0, 0x9E3779B9, 0), (2, 0, 0, 40), (3, 2, 0, 60)])
def test_sharded_protocol_equals_oracle(tmp_path, world, max_rounds, tie_seed, fold_n):
    """fold_n > 0: the sharded levels until the coarse graph has <= fold_n vertices, then the
    gathered graph (re-sharded onto rank 0) for the rest: the same hierarchy."""
    import oracle

    port = _free_port()
    mp.start_processes(_worker, args=(world, port, str(tmp_path), 8, max_rounds, tie_seed, fold_n), nprocs=world,
                       join=True,
                       start_method="spawn")
    errs = [p for p in os.listdir(tmp_path) if p.startswith("error")]
    assert not errs, open(os.path.join(tmp_path, errs[0])).read()
    import pickle
    with open(os.path.join(tmp_path, "result.pkl"), "rb") as f:
        res = pickle.load(f)
    for name, g in _graphs().items():
        g = {k: (v.numpy() if hasattr(v, "numpy") else v) for k, v in g.items()}
        ref = oracle.coarsen_to(g, threshold=8, max_rounds=max_rounds, tie_seed=tie_seed)
        pieces = res[name]
        assert all(len(p) == len(ref) for p in pieces), name
        for i, r in enumerate(ref):
            got = _concat(pieces, i)
            where = f"{name} G={world} level {i}"
            assert got["rounds"] == r["rounds"], where
            assert got["maximal"] == r["maximal"], where
            assert np.array_equal(got["match"], r["match"]), where
            assert np.array_equal(got["cmap"], r["cmap"]), where
            assert got["n_coarse"] == len(r["coarse"]["vwgt"]), where
            for k in ("adjp", "adjncy", "adjwgt", "vwgt"):
                assert np.array_equal(got["coarse"][k], np.asarray(r["coarse"][k])), f"{where} {k}"
