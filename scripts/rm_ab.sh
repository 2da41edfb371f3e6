#!/bin/bash
# quick A/B after a change of the tie-priority code: RM + small parity tests, C3 step time
# (default rule) and the RM step times of C1 / C4
mkdir -p gpurun_out
TAG=${1:-ab}
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
timeout 900 python -m pytest tests/test_rm_ties.py tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -3
for i in 1 2; do timeout 600 python bench.py --config C3 --no-cpu-baseline > gpurun_out/bench_${TAG}_C3_$i.json 2>/dev/null; done
timeout 300 python bench.py --config C1 --steps 20 --no-cpu-baseline --tie-seed 0x9e3779b9 > gpurun_out/bench_${TAG}_C1_rm.json 2>/dev/null
timeout 600 python bench.py --config C4 --steps 5 --no-cpu-baseline --tie-seed 0x9e3779b9 > gpurun_out/bench_${TAG}_C4_rm.json 2>/dev/null
for f in gpurun_out/bench_${TAG}_*.json; do echo $f; python -c "
import json; d=json.load(open('$f')); print(d['ms_per_step'], d['kernels']['match']['ms_per_step'], d['config']['rounds'][:4], d['value'])"; done
