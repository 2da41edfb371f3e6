#!/bin/bash
# per-round outcome profile (GP_PROF=1) of one config: live, slowest warp, matched / kept / second / rescanned
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
for C in ${@:-C3 C4}; do echo "== $C"; GP_DEBUG=1 GP_PROF=1 timeout 300 python -u scripts/trace_levels.py $C 2>&1 | grep -E "level|per round" | grep -v "enqueue\|reported" | tail -12 | sed "s/| match us.*//" | cut -c1-900; done
