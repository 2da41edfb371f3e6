"""Small step-by-step checks of the CUDA path with progress output (run under timeout)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen as G  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_goodarzibg16_b200.gp as gp  # noqa: E402
from gpu_helpers import assert_levels_equal, gpu_coarsen  # noqa: E402

ctx = gp.Context(0)
for name, g in [("path6", G.from_edge_list(6, [(i, i + 1, 1) for i in range(5)])),
                ("grid8", G.grid2d(8, 8)), ("del96", G.delaunay_like(96)), ("del300", G.delaunay_like(300)),
                ("rmat12", G.rmat(12)), ("road256", G.road_like(256))]:
    t = time.time()
    ref = oracle.coarsen_to(g, 100)
    got = gpu_coarsen(gp, ctx, g, 100)
    try:
        assert_levels_equal(got, ref, name)
        print("==", name, "OK", len(got), "levels", round(time.time() - t, 2), "s", flush=True)
    except AssertionError as e:
        print("==", name, "FAIL", e, flush=True)
