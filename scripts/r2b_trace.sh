#!/bin/bash
# per-level / per-phase device traces of C3 (and optionally other configs)
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
for C in ${CONFIGS:-C3}; do
GP_DEBUG=1 timeout 300 python -u scripts/trace_levels.py $C > gpurun_out/trace_${C}_plain.txt 2>&1
GP_DEBUG=1 GP_PROF=1 timeout 300 python -u scripts/trace_levels.py $C > gpurun_out/trace_${C}_prof.txt 2>&1
done
echo done
