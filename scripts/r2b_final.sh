#!/bin/bash
# Round-2 (second session) evidence set, run under gpurun: GPU tests + smoke, ncu launch list of C3
# + full captures (level-0 match / contract, the grid tail k_part), bench lines of every config and
# mode, the reference arm, loopback, sanitizer runs of the new kernels.  Outputs in gpurun_out/.
mkdir -p gpurun_out/sanitizer
TAG=${TAG:-r2b}
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
if [ -z "$SKIP_TESTS" ]; then
  timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_tests_$TAG.txt 2>&1; echo "tests rc=$? $(tail -1 gpurun_out/gpu_tests_$TAG.txt)"
  python -u -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/smoke_$TAG.txt 2>&1; echo "smoke: $(tail -2 gpurun_out/smoke_$TAG.txt | head -1)"
fi
bash scripts/ncu_launches.sh C3 $TAG > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:k_part -c 1 \
    -o gpurun_out/prof_C3_${TAG}_k_part python scripts/profile_once.py C3 > gpurun_out/prof_C3_${TAG}_k_part.log 2>&1
python scripts/summarize_profiles.py gpurun_out/ncu_summary_C3_$TAG.md gpurun_out/launches_C3_$TAG.csv \
    gpurun_out/prof_C3_${TAG}_k_match_level.ncu-rep gpurun_out/prof_C3_${TAG}_k_contract_level.ncu-rep \
    gpurun_out/prof_C3_${TAG}_k_part.ncu-rep --traffic gpurun_out/ncu_traffic_C3_$TAG.json > /dev/null 2>&1
mkdir -p profiles/r2 && cp gpurun_out/ncu_traffic_C3_$TAG.json profiles/r2/ncu_traffic_C3.json
for K in k_contract_level k_match_level k_part; do python scripts/ncu_lines.py gpurun_out/prof_C3_${TAG}_$K.ncu-rep 45 > gpurun_out/lines_${TAG}_$K.txt 2>&1; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
    --log-file gpurun_out/bench_launches_C3_$TAG.csv \
    python bench.py --config C3 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_under_ncu_$TAG.log 2>&1
timeout 900 python bench.py --config C3 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "C3: $(tail -c 200 gpurun_out/bench_$TAG.json)"
timeout 300 python bench.py --impl reference --config C3 --steps 2 --warmup 3 > gpurun_out/bench_ref_$TAG.json 2> gpurun_out/bench_ref_$TAG.err
for C in C1 C2 C5; do timeout 900 python bench.py --config $C --steps 100 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${TAG}_$C.json 2> gpurun_out/bench_${TAG}_$C.err; done
timeout 900 python bench.py --config C4 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${TAG}_C4.json 2> gpurun_out/bench_${TAG}_C4.err
for C in C2 C3 C5; do timeout 900 python bench.py --config $C --steps 20 --warmup 3 --max-rounds 1 --no-cpu-baseline > gpurun_out/bench_${TAG}_${C}_oneshot.json 2> gpurun_out/bench_${TAG}_${C}_oneshot.err; done
timeout 900 python bench.py --config C1 --steps 400 --warmup 3 --tie-seed 0x9e3779b9 --no-cpu-baseline > gpurun_out/bench_${TAG}_C1_rm.json 2> gpurun_out/bench_${TAG}_C1_rm.err
timeout 900 python bench.py --config C4 --steps 3 --warmup 3 --tie-seed 0x9e3779b9 --no-cpu-baseline > gpurun_out/bench_${TAG}_C4_rm.json 2> gpurun_out/bench_${TAG}_C4_rm.err
for G in 2 4 8; do timeout 900 python bench.py --config C3 --steps 5 --warmup 3 --loopback $G --no-cpu-baseline > gpurun_out/loopback_${TAG}_C3_G$G.json 2> gpurun_out/loopback_${TAG}_C3_G$G.err; done
for c in; do for t in memcheck; do
  timeout 900 compute-sanitizer --tool $t --print-limit 50 python scripts/sanitize_cases.py $c > gpurun_out/sanitizer/${t}_${c}.log 2>&1
  echo "$t $c rc=$? $(tail -1 gpurun_out/sanitizer/${t}_${c}.log)"
done; done
ls gpurun_out | wc -l
