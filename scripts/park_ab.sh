#!/bin/bash
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
GP_MATCH_PARK=1 timeout 180 python -u scripts/debug_small.py 2>&1 | grep -E "==|Error|error" | head -12
bash scripts/ab_env.sh C3 GP_MATCH_PARK=1 GP_MATCH_PARK=0
for P in 1 0; do echo "== C4 PARK=$P"; GP_MATCH_PARK=$P GP_DEBUG=1 timeout 300 python -u scripts/trace_levels.py C4 2>&1 | grep -E "level|rep 2" | grep -v "enqueue\|reported" | tail -4 | sed "s/| match us.*| contract/| contract/" | cut -c1-200; done
