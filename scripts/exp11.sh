python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
timeout 180 python -u scripts/debug_small.py 2>&1 | grep -E "==|Error|error" | head -12
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q 2>&1 | tail -3
bash scripts/ab_env.sh C3 X=1
GP_DEBUG=1 timeout 300 python -u scripts/trace_levels.py C4 2>&1 | grep -E "level|rep" | grep -v "enqueue\|reported" | tail -4 | sed "s/match us.*| contract/contract/"
timeout 900 python -m pytest tests/test_gpu_full.py -x -q -k rmat 2>&1 | tail -3
