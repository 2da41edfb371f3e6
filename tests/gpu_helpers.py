"""Helpers of the -m gpu parity tests: run the CUDA path through the C ABI and compare it
with the oracle element by element (bit-exact: every quantity on the path is an integer)."""
from __future__ import annotations

from typing import Dict, List

import numpy as np
import torch

import oracle


def to_device(g: Dict) -> Dict:
    return {k: (g[k].cuda() if isinstance(g[k], torch.Tensor) else torch.as_tensor(g[k]).cuda())
            for k in ("adjp", "adjncy", "adjwgt", "vwgt")}


def gpu_coarsen(gp, ctx, g: Dict, threshold: int, validate: bool = False, **kw) -> List[Dict]:
    d = to_device(g)
    G = gp.Graph.create(ctx, d["adjp"], d["adjncy"], d["adjwgt"], d["vwgt"], validate=validate)
    H = G.coarsen_to(threshold, **kw)
    out = []
    for i, info in enumerate(H.levels()):
        m, c = H.download_level(i)
        coarse = H.download_coarse(i)
        out.append({"n": info.n, "nnz": info.nnz, "n_coarse": info.n_coarse, "rounds": info.rounds,
                    "maximal": info.maximal, "stop_reason": info.stop_reason, "match": m.numpy(),
                    "cmap": c.numpy(), "coarse": {k: coarse[k].numpy() for k in ("adjp", "adjncy", "adjwgt", "vwgt")},
                    "arcs_scanned": info.arcs_scanned})
    H.close()
    G.close()
    return out


def assert_levels_equal(gpu: List[Dict], ref: List[Dict], name: str = "") -> None:
    assert len(gpu) == len(ref), f"{name}: {len(gpu)} levels on GPU vs {len(ref)} in the oracle"
    for i, (a, b) in enumerate(zip(gpu, ref)):
        where = f"{name} level {i}"
        assert a["n"] == b["n"] and a["nnz"] == b["nnz"], where
        assert a["rounds"] == b["rounds"], f"{where}: rounds {a['rounds']} vs {b['rounds']}"
        assert a["maximal"] == b["maximal"], where
        assert a["stop_reason"] == b["stop_reason"], where
        assert np.array_equal(a["match"], b["match"]), f"{where}: match differs at " \
            f"{np.nonzero(a['match'] != b['match'])[0][:10]}"
        assert np.array_equal(a["cmap"], b["cmap"]), f"{where}: cmap differs"
        assert a["n_coarse"] == b["n_coarse"], where
        for k in ("adjp", "adjncy", "adjwgt", "vwgt"):
            x, y = a["coarse"][k], b["coarse"][k]
            assert len(x) == len(y) and np.array_equal(x, y), f"{where}: coarse {k} differs"
