python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
timeout 60 python -u scripts/dbg_case.py 5000 10000 5 5 2>&1 | tail -3
timeout 300 compute-sanitizer --tool memcheck python -u scripts/dbg_case.py 5000 10000 5 5 2>&1 | grep -v "^=========     Host Frame" | head -40
