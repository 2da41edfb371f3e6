#!/bin/bash
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
GP_DEBUG=1 timeout 900 python -u scripts/trace_levels.py C4 > gpurun_out/trace_C4.txt 2>&1
grep "contract us" gpurun_out/trace_C4.txt | tail -3 | cut -c1-400
