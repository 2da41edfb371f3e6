# bench lines (1 GPU) for the configs given as args (default C3), plus optional loopback runs
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
TAG=${TAG:-r2}
for C in ${CONFIGS:-C3}; do
  timeout 900 python bench.py --config $C --steps ${STEPS:-50} --warmup 3 ${BENCH_ARGS} > gpurun_out/bench_${TAG}_$C.json 2> gpurun_out/bench_${TAG}_$C.err
  echo "$C rc=$? $(python -c "import json,sys; d=json.loads(open('gpurun_out/bench_${TAG}_$C.json').read().strip().splitlines()[-1]); print(d['ms_per_step'], d['value'], d.get('level0'), d['clocks'])" 2>&1 | tail -1)"
done
