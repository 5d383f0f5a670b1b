#!/bin/bash
# A/B: full-width scalar-column stage tiles (STENCIL_FULLW) and 5-row stage tiles on C2's TB-RT;
# parity of the TB-RT tests with FULLW forced on
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
STENCIL_FULLW=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py -m gpu -x -q \
  -k "tb_rt or every_oc or edge_every_oc or full_grid" > gpurun_out/fullw_parity.log 2>&1; echo "rc=$?" >> gpurun_out/fullw_parity.log
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 10 --top 16 \
  --grid '{"bx":[64],"by":[8],"vx":[2],"merge":[4],"pr_stages":[3,4],"tb_steps":[2],"env:FULLW":[0,1],"env:MID_ROWS":[4,5],"env:XSHIFT":[0]}' \
  > gpurun_out/ab_fullw_c2.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 10 --top 16 \
  --grid '{"bx":[64],"by":[8],"vx":[2],"merge":[4],"pr_stages":[4],"tb_steps":[2],"env:FULLW":[0,1],"env:MID_ROWS":[4,5],"env:XSHIFT":[0]}' \
  > gpurun_out/ab_fullw_c2_rep.log 2>&1
timeout 600 python scripts/dev_tune.py --cfg C5 --stencil random3d:1:0 --ocs ST_TB_BM_RT_PR --steps 4 --top 16 \
  --grid '{"bx":[64],"by":[8],"vx":[2],"merge":[4],"pr_stages":[4],"tb_steps":[2],"env:FULLW":[0,1]}' \
  > gpurun_out/ab_fullw_c5r1.log 2>&1
