#!/bin/bash
# full ncu capture of the level-0 contraction and match kernels + launch list (C3)
mkdir -p gpurun_out
TAG=${1:-r1c}
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --profile-from-start off --csv --log-file gpurun_out/launches_C3_${TAG}.csv \
    python scripts/profile_once.py C3 > /dev/null 2>&1
for K in k_contract_level k_match_level; do
timeout 600 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:$K -c 1 \
    -o gpurun_out/prof_C3_${TAG}_$K python scripts/profile_once.py C3 > /dev/null 2>&1
done
GP_DEBUG=1 timeout 120 python -u scripts/trace_levels.py C3 2>&1 | grep -v enqueue | grep -v reported | tail -14
