#!/bin/bash
# A/B: L2 cache-policy hints in k_match_level (GP_L2HINT: evict_last on P/S gathers,
# evict_first on streamed arcs and phase-0 TMA stages), with and without an L2 set-aside
for V in base hint; do
  D=""; [ $V = hint ] && D="-DGP_L2HINT"
  GP_NVCC_DEFS="$D" python -c "from paper_conf_ipps_goodarzibg16_b200 import _build; _build.build(force=True)" > gpurun_out/build_$V.log 2>&1 || { echo BUILD FAIL; exit 1; }
  for P in 0 64; do
    [ $V = base ] && [ $P = 64 ] && continue
    for rep in 1 2; do for C in C3 C5; do
      GP_L2_PERSIST_MB=$P timeout 600 python bench.py --config $C --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/l2_${V}_${P}_$C.json 2>/dev/null
      echo "$V persist=$P rep$rep $C $(python -c "import json; d=json.loads(open('gpurun_out/l2_${V}_${P}_$C.json').read().strip().splitlines()[-1]); l=d['levels'][0]; print(d['ms_per_step'], l.get('match_us'), l.get('contract_us'))" 2>&1 | tail -1)"
    done; done
  done
done
