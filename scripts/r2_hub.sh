python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
for C in C3 C2; do
for cfg in "1024 0" "64 500000" "32 500000" "48 2000000" "16 300000"; do set -- $cfg
  r=$(GP_HUB_DEG_SMALL=$1 GP_HUB_SMALL_N=$2 timeout 300 python bench.py --config $C --steps 60 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['ms_per_step'],3))")
  echo "$C hub_deg_small=$1 n<=$2: $r ms"
done; done
GP_HUB_DEG_SMALL=32 GP_HUB_SMALL_N=500000 timeout 600 python -m pytest tests -x -q -m gpu -k "parity and (small or random or shuffled)" > gpurun_out/hub_tests.txt 2>&1; echo "tests: $(tail -1 gpurun_out/hub_tests.txt)"
