#!/bin/bash
# A/B of dev switches on one box: for each env setting (";"-separated list in
# $AB), time OCs with scripts/dev_time.py, twice in alternating order.
#   AB="STENCIL_ELECT=0;STENCIL_ELECT=1" ARGS="--cfg C2 --ocs ST_TB_BM_RT_PR" bash scripts/gpu_ab_env.sh
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
IFS=';' read -ra SET <<< "$AB"
for rep in 1 2; do
  for cfg in "${SET[@]}"; do
    echo "== [$rep] $cfg"
    env $cfg python scripts/dev_time.py $ARGS 2>&1 | grep -v Warning
  done
done
