#!/bin/bash
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_dist.py tests/test_gpu_abi.py -m gpu -q -x > gpurun_out/fold_tests.txt 2>&1; echo "tests rc=$? $(tail -1 gpurun_out/fold_tests.txt)"
bash scripts/r2_l2hint.sh
