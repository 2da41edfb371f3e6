python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
bash scripts/ab_env.sh C3 "GP_TB_MIN=128" "GP_TB_MIN=32"
GP_DEBUG=1 GP_PROF=1 timeout 120 python -u scripts/trace_levels.py C3 2>&1 | grep -E "barriers|level|per round" | grep -v enqueue | grep -v reported | tail -36 | sed "s/| contract us.*//" | cut -c1-330
