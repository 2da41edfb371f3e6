GP_NVCC_DEFS=-DGP_CHECKPOINTS python -c "from paper_conf_ipps_goodarzibg16_b200 import _build; _build.build(force=True)" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; exit 1; }
GP_DEBUG=1 GP_PROF=2 timeout 300 python -u scripts/trace_levels.py C3 > gpurun_out/ck_C3.txt 2>&1
GP_DEBUG=1 GP_PROF=2 timeout 300 python -u scripts/trace_levels.py C1 > gpurun_out/ck_C1.txt 2>&1
grep -c checkpoints gpurun_out/ck_C3.txt
