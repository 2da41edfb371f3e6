python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
for rep in 1 2; do for C in C3 C2 C5; do
for mv in 256 512 768 1024; do for cv in 64 128 256; do
  [ $C = C5 ] && [ $cv != 128 ] && continue
  r=$(GP_MATCH_VPC=$mv GP_CONTRACT_VPC=$cv timeout 300 python bench.py --config $C --steps 60 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['ms_per_step'],3))")
  echo "rep$rep $C match_vpc=$mv contract_vpc=$cv: $r ms"
done; done; done; done
