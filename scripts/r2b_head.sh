#!/bin/bash
# HEAD check after re-entry: build, GPU tests, smoke, C3/C4 bench lines
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_tests_head.txt 2>&1; echo "tests rc=$? $(tail -1 gpurun_out/gpu_tests_head.txt)"
python -u -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/smoke_head.txt 2>&1; echo "smoke: $(tail -2 gpurun_out/smoke_head.txt | head -1)"
timeout 900 python bench.py --config C3 > gpurun_out/bench_head_C3.json 2> gpurun_out/bench_head_C3.err; echo "C3: $(tail -c 400 gpurun_out/bench_head_C3.json)"
timeout 900 python bench.py --config C4 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_head_C4.json 2> gpurun_out/bench_head_C4.err; echo "C4: $(head -c 300 gpurun_out/bench_head_C4.json)"
