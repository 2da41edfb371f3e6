#!/bin/bash
# Sweep the active-CTA knobs of the level kernels (results never depend on them):
#   GP_MATCH_VPC / GP_CONTRACT_VPC = vertices per active CTA.  Prints step time per setting.
mkdir -p gpurun_out
CFG=${1:-C3}
timeout 120 python -u -c "import __graft_entry__ as e; e.build(); e.smoke()" 2>&1 | tail -1
for mv in ${MVS:-128 1024}; do
  for cv in ${CVS:-64 512}; do
    echo "== match_vpc=$mv contract_vpc=$cv"
    GP_MATCH_VPC=$mv GP_CONTRACT_VPC=$cv timeout 120 python -u scripts/trace_levels.py $CFG 2>&1 | grep "rep 2"
  done
done
GP_DEBUG=1 timeout 120 python -u scripts/trace_levels.py $CFG 2>&1 | grep -v enqueue | grep -v reported | tail -13 | cut -c1-330
