for B in 4 3; do
GP_NVCC_DEFS=-DGP_CONTRACT_MINB=$B python -c "from paper_conf_ipps_goodarzibg16_b200 import _build; _build.build(force=True)" > gpurun_out/build_$B.log 2>&1 || { echo BUILD FAIL; exit 1; }
for rep in 1 2; do for C in C3 C2 C5; do
  r=$(timeout 300 python bench.py --config $C --steps 60 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['ms_per_step'],3), round(d['level0']['contract_us'],1))")
  echo "minB=$B rep$rep $C: $r"
done; done; done
