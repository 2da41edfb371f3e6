#!/bin/bash
# Memory-safety check of the grid tail (compute-sanitizer is closed on this pool): build with
# -DGP_PART_CHECK (every shared / staging / output index of k_part range-checked, a violation
# prints and traps) and run the GPU parity suites that exercise k_part, plus C2 / C3 / C5 at
# full size.  Outputs in gpurun_out/part_checked_*.txt.
rm -f paper_conf_ipps_goodarzibg16_b200/lib/libgpcoarsen.so
GP_NVCC_DEFS="-DGP_PART_CHECK" python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build_checked.log 2>&1 || { echo BUILD FAIL; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_tail.py tests/test_gpu_parity.py tests/test_gpu_dist.py tests/test_rm_ties.py tests/test_refine.py -m gpu -q > gpurun_out/part_checked_suites.txt 2>&1
echo "suites rc=$? $(tail -1 gpurun_out/part_checked_suites.txt)"
timeout 900 python -m pytest tests/test_gpu_full.py -m gpu -q -k "C2 or C3 or C5" > gpurun_out/part_checked_full.txt 2>&1
echo "full rc=$? $(tail -1 gpurun_out/part_checked_full.txt)"
timeout 600 python -u scripts/part_check.py > gpurun_out/part_checked_cases.txt 2>&1
echo "cases: $(grep -c OK gpurun_out/part_checked_cases.txt) OK, $(grep -c FAIL gpurun_out/part_checked_cases.txt) FAIL"
grep -h "check failed" gpurun_out/part_checked_*.txt | head -5
rm -f paper_conf_ipps_goodarzibg16_b200/lib/libgpcoarsen.so
