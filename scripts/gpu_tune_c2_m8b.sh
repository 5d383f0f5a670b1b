#!/bin/bash
# C2 TB-RT around (merge 8, by 4, full-width stage tiles): stage tile rows, planes in flight, stage-ring slots
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 10 --top 20 \
  --grid '{"bx":[64],"by":[4],"vx":[2],"merge":[8],"pr_stages":[3,4,6],"tb_steps":[2],"env:FULLW":[1],"env:MID_ROWS":[5,9],"env:XSHIFT":[0],"env:MIDR":[2,3]}' \
  > gpurun_out/tune_c2_m8b.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C5 --stencil random3d:1:0 --ocs ST_TB_BM_RT_PR --steps 4 --top 20 \
  --grid '{"bx":[64],"by":[4,8],"vx":[2],"merge":[4,8],"pr_stages":[4],"tb_steps":[2],"env:FULLW":[0,1],"env:MID_ROWS":[5]}' \
  > gpurun_out/tune_c5r1_m8.log 2>&1
