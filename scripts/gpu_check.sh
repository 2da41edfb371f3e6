#!/bin/bash
# one GPU round-trip with hard timeouts: debug parity, smoke, GPU tests, a short bench, trace
mkdir -p gpurun_out
timeout 180 python -u scripts/debug_small.py 2>&1 | grep -E "==|Error|error" | head -12
timeout 120 python -u -c "import __graft_entry__ as e; e.build(); e.smoke()" 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_full.py::test_full_rmat_s24 2>&1 | tail -15
timeout 300 python -u bench.py --steps 10 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-1500
GP_DEBUG=1 timeout 120 python -u scripts/trace_levels.py C3 2>&1 | grep -v enqueue | grep -v reported | tail -13 | sed "s/ | c2 tiles.*//" | cut -c1-330
