#!/bin/bash
# A/B of env knobs on one config: bash scripts/ab_env.sh CFG "VAR=a VAR2=b" "VAR=c" ...
# prints "rep 2" step times (3 runs each) per setting
CFG=$1; shift
for setting in "$@"; do
  echo "== $setting"
  for i in 1 2 3; do env $setting timeout 120 python -u scripts/trace_levels.py $CFG 2>&1 | grep "rep 2"; done
done
