# loopback (simulated sharded protocol on 1 GPU) step times: protocol-overhead estimate
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
for C in ${CONFIGS:-C3}; do for G in ${LOOPS:-2 4 8}; do
  timeout 900 python bench.py --config $C --steps ${STEPS:-5} --warmup 3 --loopback $G --no-cpu-baseline > gpurun_out/loopback_${C}_G$G.json 2> gpurun_out/loopback_${C}_G$G.err
  echo "$C G=$G rc=$? $(python -c "import json; d=json.loads(open('gpurun_out/loopback_${C}_G$G.json').read().strip().splitlines()[-1]); print(d['ms_per_step'])" 2>&1 | tail -1)"
done; done
