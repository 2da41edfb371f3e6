#!/bin/bash
# folding on the sharded path: GPU tests of the loopback / NCCL paths, loopback C3 timings with
# folding off and at the default limit, and the contraction instantiation A/B on C3/C2/C4/C5
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; tail gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_dist.py tests/test_gpu_abi.py tests/test_rm_ties.py -m gpu -q -x > gpurun_out/fold_tests.txt 2>&1; echo "tests rc=$? $(tail -1 gpurun_out/fold_tests.txt)"
for G in 2 8; do for F in 0 500000; do
  GP_FOLD_N=$F timeout 600 python bench.py --config C3 --steps 5 --warmup 3 --loopback $G --no-cpu-baseline > gpurun_out/lb_G${G}_F$F.json 2> gpurun_out/lb_G${G}_F$F.err
  echo "G=$G fold=$F $(python -c "import json,sys; d=json.loads(open('gpurun_out/lb_G${G}_F$F.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['value'])" 2>&1 | tail -1)"
done; done
for C in C3 C2 C5 C4; do for B in 0 3 4; do
  ST=20; [ $C = C4 ] && ST=3
  GP_CONTRACT_MINB=$B timeout 600 python bench.py --config $C --steps $ST --warmup 3 --no-cpu-baseline > gpurun_out/mb_${C}_$B.json 2>/dev/null
  echo "$C minB=$B $(python -c "import json; d=json.loads(open('gpurun_out/mb_${C}_$B.json').read().strip().splitlines()[-1]); print(d['ms_per_step'])" 2>&1 | tail -1)"
done; done
