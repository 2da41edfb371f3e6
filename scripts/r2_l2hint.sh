#!/bin/bash
# A/B: L2 cache-policy hints in k_match_level.  GP_L2HINT=1: evict_first on streamed arcs and
# phase-0 TMA stages; =2: also evict_last on the P/S gathers
for V in 0 1 2; do
  D=""; [ $V != 0 ] && D="-DGP_L2HINT=$V"
  GP_NVCC_DEFS="$D" python -c "from paper_conf_ipps_goodarzibg16_b200 import _build; _build.build(force=True)" > gpurun_out/build_$V.log 2>&1 || { echo BUILD FAIL; exit 1; }
  for rep in 1 2; do for C in C3 C2 C5; do
    timeout 600 python bench.py --config $C --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/l2_${V}_$C.json 2>/dev/null
    echo "hint=$V rep$rep $C $(python -c "import json; d=json.loads(open('gpurun_out/l2_${V}_$C.json').read().strip().splitlines()[-1]); l=d['levels'][0]; print(d['ms_per_step'], l.get('match_us'), l.get('contract_us'))" 2>&1 | tail -1)"
  done; done
done
