python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; tail gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_tail.py -x -q -m gpu > gpurun_out/tail_tests.txt 2>&1; echo "tail tests rc=$? $(tail -1 gpurun_out/tail_tests.txt)"
mkdir -p gpurun_out/sanitizer; for c in c1_tail medium_tail; do timeout 600 compute-sanitizer --tool racecheck python scripts/sanitize_cases.py $c > gpurun_out/sanitizer/racecheck_$c.log 2>&1; echo "racecheck $c: $(tail -1 gpurun_out/sanitizer/racecheck_$c.log)"; done
for C in C3 C2; do GP_DEBUG=1 timeout 300 python -u scripts/trace_levels.py $C 2>&1 | grep "rep\|level" | grep -v "reported\|enqueue" > gpurun_out/trace_tail_$C.txt; grep rep gpurun_out/trace_tail_$C.txt; done
