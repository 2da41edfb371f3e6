#!/bin/bash
# full GPU test suite + smoke + round profile (bench, reference arm, ncu launch lists, L0 captures)
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
TAG=${1:-r1f}
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 > gpurun_out/gpu_tests_$TAG.txt
python -u -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/smoke_$TAG.txt 2>&1
bash scripts/profile_round.sh $TAG C3 > gpurun_out/profile_round_$TAG.log 2>&1
for K in k_contract_level k_match_level; do python scripts/ncu_lines.py gpurun_out/prof_C3_${TAG}_$K.ncu-rep 45 > gpurun_out/lines_${TAG}_$K.txt 2>&1; done
for C in C1 C2 C4 C5; do timeout 600 python bench.py --config $C --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${TAG}_$C.json 2> gpurun_out/bench_${TAG}_$C.err; done
cat gpurun_out/gpu_tests_$TAG.txt gpurun_out/smoke_$TAG.txt; tail -c 1500 gpurun_out/bench_$TAG.json
