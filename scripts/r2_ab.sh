# A/B of match knobs on C3 / C1: per-level traces
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
for L in 1 2; do
  GP_MATCH_LANES=$L GP_DEBUG=1 timeout 300 python -u scripts/trace_levels.py C3 > gpurun_out/trace_C3_lanes$L.txt 2>&1
  GP_MATCH_LANES=$L GP_DEBUG=1 timeout 300 python -u scripts/trace_levels.py C1 > gpurun_out/trace_C1_lanes$L.txt 2>&1
  echo "lanes=$L C3: $(grep rep gpurun_out/trace_C3_lanes$L.txt | tr '\n' ' ')  C1: $(grep rep gpurun_out/trace_C1_lanes$L.txt | tr '\n' ' ')"
done
GP_MATCH_LANES=2 timeout 900 python -m pytest tests -x -q -m gpu -k "parity or modes or rm_ties" > gpurun_out/gpu_tests_lanes2.txt 2>&1; echo "lanes2 tests rc=$?"; tail -3 gpurun_out/gpu_tests_lanes2.txt
