# compute-sanitizer evidence for the lock-free / grid-barrier protocols (profiles/r2/sanitizer/)
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
mkdir -p gpurun_out/sanitizer
for c in c3_256 star5000 loopback3; do
  for t in memcheck racecheck synccheck; do
    timeout 900 compute-sanitizer --tool $t --print-limit 50 python scripts/sanitize_cases.py $c > gpurun_out/sanitizer/${t}_${c}.log 2>&1
    echo "$t $c rc=$? $(tail -2 gpurun_out/sanitizer/${t}_${c}.log | tr '\n' ' ')"
  done
done
