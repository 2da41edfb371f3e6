#!/bin/bash
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; tail -20 gpurun_out/build.log; exit 1; }
timeout 600 python -u scripts/part_check.py $@ 2>&1 | tail -40
GP_DEBUG=1 timeout 120 python -u scripts/trace_levels.py C3 > gpurun_out/trace_C3_part.txt 2>&1
grep -E "^\[gp\] level [0-9]+ n=" gpurun_out/trace_C3_part.txt | tail -12 | cut -c1-200
