#!/bin/bash
# part kernel iteration: build, parity subset, C3/C2 A/B, per-round slowest CTA (GP_PROF)
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; tail -20 gpurun_out/build.log; exit 1; }
timeout 600 python -u scripts/part_check.py ${CASES:-grid40 rmat10 star5000 delaunay512} 2>&1 | grep -v "^C3" | tail -14
python scripts/part_ab.py C3 2>&1 | tail -2
python scripts/part_ab.py C2 2>&1 | tail -2
GP_DEBUG=1 GP_PROF=1 timeout 120 python -u scripts/trace_levels.py C3 > gpurun_out/trace_C3_partprof.txt 2>&1
grep -E "part:|per round \(live" gpurun_out/trace_C3_partprof.txt | tail -14 | cut -c1-250
