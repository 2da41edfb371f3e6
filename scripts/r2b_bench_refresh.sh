#!/bin/bash
# final bench lines of this session's build (profiles/r2b/bench): C3 (default line), C4, C4 RM, C2, C1
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
TAG=r2b
timeout 900 python bench.py --config C3 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "C3 rc=$?"
timeout 900 python bench.py --config C4 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${TAG}_C4.json 2> gpurun_out/bench_${TAG}_C4.err; echo "C4 rc=$?"
timeout 900 python bench.py --config C4 --steps 3 --warmup 3 --tie-seed 0x9e3779b9 --no-cpu-baseline > gpurun_out/bench_${TAG}_C4_rm.json 2> gpurun_out/bench_${TAG}_C4_rm.err; echo "C4rm rc=$?"
for C in C1 C2; do timeout 900 python bench.py --config $C --steps 100 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${TAG}_$C.json 2> gpurun_out/bench_${TAG}_$C.err; echo "$C rc=$?"; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
    --log-file gpurun_out/bench_launches_C3_$TAG.csv \
    python bench.py --config C3 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_under_ncu_$TAG.log 2>&1
echo done
