M=paper_conf_ipps_goodarzibg16_b200/csrc/match.cu
C=paper_conf_ipps_goodarzibg16_b200/csrc/contract.cu
cp $M /tmp/m.cu; cp $C /tmp/c.cu
run() { python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1 || { echo BUILD FAIL; return; }; timeout 60 python -u scripts/dbg_case.py 5000 10000 5 5 2>&1 | tail -1; timeout 60 python -u scripts/dbg_case.py 1000 8000 12 5 2>&1 | tail -1; }
gen() { sed -i 's|MatchSmem \&sm = \*reinterpret_cast<MatchSmem \*>(smem_raw + .*|MatchSmem \&sm = *reinterpret_cast<MatchSmem *>(((uintptr_t)smem_raw + 127) \& ~(uintptr_t)127);|' $M; }
genc() { sed -i 's|ContractSmem \&sm = \*reinterpret_cast<ContractSmem \*>(smem_raw + .*|ContractSmem \&sm = *reinterpret_cast<ContractSmem *>(((uintptr_t)smem_raw + 127) \& ~(uintptr_t)127);|' $C; }
echo "== D both generic (flat32 kept)"; gen; genc; run
cp /tmp/m.cu $M; cp /tmp/c.cu $C
echo "== E head match + smem fix, contract new"; cp scripts/tmpv/match_head.cu $M; run
echo "== F head match + smem fix, contract generic"; genc; run
cp /tmp/m.cu $M; cp /tmp/c.cu $C
