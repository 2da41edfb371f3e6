#!/bin/bash
# RM tie mode (DESIGN R17) on the GPU: seeded parity tests, the whole GPU suite after the
# key change, C3 bench (default rule, must not regress) + its ncu launch list, and the
# default-vs-RM step times of the tie-heavy configs (C1 unit grid, C4 R-MAT [1,4]).
mkdir -p gpurun_out
TAG=${1:-r1i}
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
timeout 900 python -m pytest tests/test_rm_ties.py -m gpu -q -x 2>&1 | tail -3 > gpurun_out/rm_tests_$TAG.txt
cat gpurun_out/rm_tests_$TAG.txt
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 > gpurun_out/gpu_tests_$TAG.txt
python -u -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/smoke_$TAG.txt 2>&1
cat gpurun_out/gpu_tests_$TAG.txt gpurun_out/smoke_$TAG.txt
timeout 600 python bench.py --config C3 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
    --log-file gpurun_out/bench_launches_C3_$TAG.csv \
    python bench.py --config C3 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_under_ncu_$TAG.log 2>&1
for C in C1 C4 C2 C5; do
  for S in 0 0x9e3779b9; do
    timeout 600 python bench.py --config $C --steps 5 --warmup 3 --no-cpu-baseline --tie-seed $S \
      > gpurun_out/bench_${TAG}_${C}_seed$S.json 2> gpurun_out/bench_${TAG}_${C}_seed$S.err
  done
done
tail -c 600 gpurun_out/bench_$TAG.json
for f in gpurun_out/bench_${TAG}_C*_seed*.json; do echo $f; python -c "
import json,sys; d=json.load(open('$f')); c=d['config']; print(d['ms_per_step'], c['levels'], c['rounds'][:6], d['value'])"; done
