#!/bin/bash
# Round profile set (run under gpurun; results land in gpurun_out/, summarised into profiles/<tag>/):
#   1. bench.py (default run incl. cpu_baseline) and the reference arm -> bench_<tag>.json, bench_ref_<tag>.json
#   2. ncu launch list of the bench command itself (gpu__time_duration, --clock-control none)
#   3. ncu launch list + DRAM bytes of one clean gp_coarsen_to, and full captures of the L0 kernels
mkdir -p gpurun_out
TAG=${1:-r1}
CFG=${2:-C3}
timeout 600 python bench.py --config $CFG > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
timeout 300 python bench.py --impl reference --config $CFG --steps 2 --warmup 3 > gpurun_out/bench_ref_${TAG}.json 2> gpurun_out/bench_ref_${TAG}.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
    --log-file gpurun_out/bench_launches_${CFG}_${TAG}.csv \
    python bench.py --config $CFG --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_under_ncu_${TAG}.log 2>&1
bash scripts/ncu_launches.sh $CFG $TAG
tail -c 3000 gpurun_out/bench_${TAG}.json; tail -c 1500 gpurun_out/bench_ref_${TAG}.json; tail -3 gpurun_out/bench_${TAG}.err
ls -la gpurun_out
