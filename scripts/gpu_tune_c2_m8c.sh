#!/bin/bash
# C2 TB-RT 8-row setting: planes in flight, stage-ring slots, elected-lane arrivals
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 10 --top 20 \
  --grid '{"bx":[64],"by":[4],"vx":[2],"merge":[8],"pr_stages":[4,5],"tb_steps":[2],"env:MIDR":[3,4],"env:ELECT":[0,1]}' \
  > gpurun_out/tune_c2_m8c.log 2>&1
