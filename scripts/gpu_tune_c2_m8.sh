#!/bin/bash
# C2 TB-RT: 8-row last-stage tiles (merge 8, by 4: the same 64 x 32 output tile with 4 last-stage warps)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 10 --top 16 \
  --grid '{"bx":[64],"by":[4,8],"vx":[2],"merge":[4,8],"pr_stages":[4],"tb_steps":[2],"env:FULLW":[0,1],"env:MID_ROWS":[4,5],"env:XSHIFT":[0]}' \
  > gpurun_out/tune_c2_m8.log 2>&1
