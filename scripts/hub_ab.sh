#!/bin/bash
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
timeout 180 python -u scripts/debug_small.py 2>&1 | grep -E "==|Error|error" | head -12
bash scripts/ab_env.sh C3 X=1
for C in C4 C2 C5; do echo "== $C"; timeout 300 python -u scripts/trace_levels.py $C 2>&1 | grep -E "rep 2"; done
