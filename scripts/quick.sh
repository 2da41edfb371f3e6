#!/bin/bash
# quick GPU iteration: build, small parity, GPU parity tests (no full-size), step time A/B, per-level trace
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; tail gpurun_out/build.log; exit 1; }
timeout 180 python -u scripts/debug_small.py 2>&1 | grep -E "==|Error|error" | head -12
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q 2>&1 | tail -3
bash scripts/ab_env.sh C3 ${AB:-X=1}
GP_DEBUG=1 GP_PROF=1 timeout 120 python -u scripts/trace_levels.py C3 2>&1 | grep -E "c2a tiles|level|per round|barriers" | grep -v "enqueue\|reported" | tail -48 | cut -c1-300 > gpurun_out/trace.txt
grep -E "^\[gp\] level" gpurun_out/trace.txt | sed "s/| gap to.*//"
