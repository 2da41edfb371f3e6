# ncu full captures of small-level match/contract kernels (latency analysis of coarse levels)
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
ncu --set full --import-source on --clock-control none -k regex:k_match_level -s 10 -c 1 -o gpurun_out/prof_C3_L10_match -f python scripts/trace_levels.py C3 > gpurun_out/ncu_small1.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_contract_level -s 10 -c 1 -o gpurun_out/prof_C3_L10_contract -f python scripts/trace_levels.py C3 > gpurun_out/ncu_small2.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_match_level -s 1 -c 1 -o gpurun_out/prof_C1_L1_match -f python scripts/trace_levels.py C1 > gpurun_out/ncu_small3.log 2>&1
ls -la gpurun_out/*.ncu-rep
