python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || exit 1
ncu --set full --import-source on --clock-control none -k regex:k_small -s 1 -c 1 -o gpurun_out/prof_k_small_C1 -f python scripts/trace_levels.py C1 > gpurun_out/ncu_k_small.log 2>&1
tail -3 gpurun_out/ncu_k_small.log
