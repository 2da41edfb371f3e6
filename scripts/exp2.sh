#!/bin/bash
python -c "import __graft_entry__ as e; e.build()" > /dev/null 2>&1 || { echo BUILD FAIL; exit 1; }
for t in 32 256; do echo "== trace TB_MIN=$t"; GP_TB_MIN=$t GP_DEBUG=1 GP_PROF=1 timeout 120 python -u scripts/trace_levels.py C3 2>&1 | grep -E "c2a tiles|contract us" | tail -24 | sed "s/| match us.*| contract/| contract/" | cut -c1-300; done
