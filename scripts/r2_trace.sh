set -x
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; tail gpurun_out/build.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
GP_DEBUG=1 timeout 300 python -u scripts/trace_levels.py C3 > gpurun_out/trace_C3.txt 2>&1
GP_DEBUG=1 GP_PROF=1 timeout 300 python -u scripts/trace_levels.py C3 > gpurun_out/trace_C3_prof.txt 2>&1
GP_DEBUG=1 timeout 300 python -u scripts/trace_levels.py C1 > gpurun_out/trace_C1.txt 2>&1
tail -5 gpurun_out/trace_C3.txt
