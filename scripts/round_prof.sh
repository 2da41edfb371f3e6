#!/bin/bash
# build + profile_round (bench, reference arm, ncu launch lists, L0 full captures) + line summaries
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
TAG=${1:-r1e}
bash scripts/profile_round.sh $TAG C3 > gpurun_out/profile_round_$TAG.log 2>&1
for K in k_contract_level k_match_level; do python scripts/ncu_lines.py gpurun_out/prof_C3_${TAG}_$K.ncu-rep 45 > gpurun_out/lines_${TAG}_$K.txt 2>&1; done
tail -c 2500 gpurun_out/bench_$TAG.json; echo; tail -c 600 gpurun_out/bench_ref_$TAG.json
