python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
timeout 300 compute-sanitizer --tool memcheck python -u scripts/dbg_case.py 100 800 3 2 2 2>&1 | grep -v "Host Frame" | head -30
