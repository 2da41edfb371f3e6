python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
bash scripts/ncu_contract.sh r1d > /dev/null 2>&1
for K in k_contract_level k_match_level; do python scripts/ncu_lines.py gpurun_out/prof_C3_r1d_$K.ncu-rep 45 > gpurun_out/lines_r1d_$K.txt 2>&1; done
ls -la gpurun_out/*r1d*
