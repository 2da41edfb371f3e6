#!/bin/bash
# full ncu captures of the match and contraction kernels of chosen levels (C3 default)
#   usage: bash scripts/ncu_levels.sh TAG "0 8" [CFG]
mkdir -p gpurun_out
TAG=${1:-x}
LEVELS=${2:-"0 8"}
CFG=${3:-C3}
python -c "import __graft_entry__ as e; e.build()" > /dev/null 2>&1
for L in $LEVELS; do
for K in k_match_level k_contract_level; do
timeout 600 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:$K \
    --launch-skip $L -c 1 -o gpurun_out/prof_${CFG}_${TAG}_${K}_L$L python scripts/profile_once.py $CFG > /dev/null 2>&1
echo "== $K L$L"; python scripts/ncu_hot.py gpurun_out/prof_${CFG}_${TAG}_${K}_L$L.ncu-rep 30
done
done
