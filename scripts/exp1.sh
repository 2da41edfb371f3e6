#!/bin/bash
# tile-budget floor A/B + per-round slowest-warp profile
python -c "import __graft_entry__ as e; e.build()" > /dev/null 2>&1 || { echo BUILD FAIL; exit 1; }
bash scripts/ab_env.sh C3 "GP_TB_MIN=32" "GP_TB_MIN=64" "GP_TB_MIN=128" "GP_TB_MIN=256"
for t in 32 256; do echo "== trace TB_MIN=$t"; GP_TB_MIN=$t GP_DEBUG=1 GP_PROF=1 timeout 120 python -u scripts/trace_levels.py C3 2>&1 | grep -v enqueue | grep -v reported | tail -25 | cut -c1-400; done
