python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x --durations=8 2>&1 | tail -15
GP_MATCH_STATIC=1 timeout 900 python -m pytest tests/test_gpu_full.py tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -3
python -u -c "import __graft_entry__ as e; e.smoke()" 2>&1 | tail -2
