"""Tuning knobs never change results (-m gpu): the small parity set (golden graphs, meshes,
R-MAT, roads; every level vs the oracle) re-run in fresh processes with each env knob of the
level kernels set -- optional static round walk, parking, no lane mode, contiguous groups.
The knobs are read once per process, hence the subprocesses."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("env", ["GP_MATCH_PARK=1", "GP_MATCH_STATIC=1", "GP_MATCH_LANES=0", "GP_MATCH_CONTIG=1",
                                 "GP_TAIL_LIVE=0", "GP_MATCH_VPC=4096"])
def test_knob_results_identical(env):
    k, v = env.split("=")
    e = dict(os.environ)
    e[k] = v
    out = subprocess.run([sys.executable, "-u", os.path.join(ROOT, "scripts", "debug_small.py")], env=e,
                         capture_output=True, text=True, timeout=600, cwd=ROOT)
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("==")]
    assert out.returncode == 0, out.stderr[-2000:]
    assert len(lines) == 6 and all(" OK " in ln for ln in lines), "\n".join(lines) + out.stderr[-2000:]
