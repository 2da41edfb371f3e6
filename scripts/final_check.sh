#!/bin/bash
# Round-end evidence set (run under gpurun): GPU tests + smoke, ncu launch lists + L0 full
# captures of C3, traffic JSON (read by bench.py), the bench line + reference arm, other configs.
mkdir -p gpurun_out
TAG=${1:-r1g}
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 > gpurun_out/gpu_tests_$TAG.txt
python -u -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/smoke_$TAG.txt 2>&1
bash scripts/ncu_launches.sh C3 $TAG > /dev/null 2>&1
python scripts/summarize_profiles.py gpurun_out/ncu_summary_C3_$TAG.md gpurun_out/launches_C3_$TAG.csv \
    gpurun_out/prof_C3_${TAG}_k_match_level.ncu-rep gpurun_out/prof_C3_${TAG}_k_contract_level.ncu-rep \
    --traffic gpurun_out/ncu_traffic_C3_$TAG.json > /dev/null 2>&1
cp gpurun_out/ncu_traffic_C3_$TAG.json profiles/r1/ncu_traffic_C3.json
for K in k_contract_level k_match_level; do python scripts/ncu_lines.py gpurun_out/prof_C3_${TAG}_$K.ncu-rep 45 > gpurun_out/lines_${TAG}_$K.txt 2>&1; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
    --log-file gpurun_out/bench_launches_C3_$TAG.csv \
    python bench.py --config C3 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_under_ncu_$TAG.log 2>&1
timeout 600 python bench.py --config C3 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
timeout 300 python bench.py --impl reference --config C3 --steps 2 --warmup 3 > gpurun_out/bench_ref_$TAG.json 2> gpurun_out/bench_ref_$TAG.err
for C in C1 C2 C4 C5; do timeout 900 python bench.py --config $C --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${TAG}_$C.json 2> gpurun_out/bench_${TAG}_$C.err; done
cat gpurun_out/gpu_tests_$TAG.txt gpurun_out/smoke_$TAG.txt; tail -c 1200 gpurun_out/bench_$TAG.json
