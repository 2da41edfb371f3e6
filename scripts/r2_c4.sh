#!/bin/bash
# C4 contraction: balanced big-tile copy + shift-indexed bitonic sorts; parity + timings
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; tail gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x -k "rmat or star or hub or C4 or c4 or contract" > gpurun_out/c4_tests.txt 2>&1; echo "tests rc=$? $(tail -1 gpurun_out/c4_tests.txt)"
GP_DEBUG=1 timeout 900 python -u scripts/trace_levels.py C4 > gpurun_out/trace_C4.txt 2>&1
grep "rounds=" gpurun_out/trace_C4.txt | tail -3 | sed 's/.*contract us/contract us/'
grep "^rep" gpurun_out/trace_C4.txt
for C in C4 C3 C5; do ST=20; [ $C = C4 ] && ST=3
  timeout 600 python bench.py --config $C --steps $ST --warmup 3 --no-cpu-baseline > gpurun_out/c4x_$C.json 2>/dev/null
  echo "$C $(python -c "import json; d=json.loads(open('gpurun_out/c4x_$C.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], [(l['match_us'], l['contract_us']) for l in d['levels'][:3]])" 2>&1 | tail -1)"
done
