#!/bin/bash
# ncu launch list (per-launch device time, cold-cache, serialised) of one profiled coarsen_to,
# plus full captures of the level-0 match and contraction kernels.  Run under gpurun.
mkdir -p gpurun_out
CFG=${1:-C3}
TAG=${2:-r1}
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --profile-from-start off --csv --log-file gpurun_out/launches_${CFG}_${TAG}.csv \
    python scripts/profile_once.py $CFG > gpurun_out/launches_${CFG}_${TAG}.log 2>&1
for K in k_match_level k_contract_level; do
timeout 600 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:$K -c 1 \
    -o gpurun_out/prof_${CFG}_${TAG}_$K python scripts/profile_once.py $CFG > gpurun_out/prof_${CFG}_${TAG}_$K.log 2>&1
done
ls gpurun_out
