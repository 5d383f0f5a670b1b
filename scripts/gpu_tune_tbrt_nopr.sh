#!/bin/bash
# TB-RT without prefetching (NS = 1) and without merging: tile shapes and 2 CTAs per SM (C2, C5 order 1)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_RT,ST_TB_BM_RT,ST_TB_CM_RT --steps 10 --top 30 \
  --grid '{"bx":[64],"by":[4,8,16],"vx":[2],"merge":[2,4],"pr_stages":[1],"tb_steps":[2],"env:MINB":[1,2]}' \
  > gpurun_out/tune_tbrt_nopr_c2.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_RT_PR --steps 10 --top 30 \
  --grid '{"bx":[64,128],"by":[4,8,16,32],"vx":[2],"merge":[1],"pr_stages":[3,4],"tb_steps":[2],"env:MINB":[1,2]}' \
  > gpurun_out/tune_tbrt_nomerge_c2.log 2>&1
