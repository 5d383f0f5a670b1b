#!/bin/bash
# C5 order-1 (3x3-plane Algorithm-1 stencil, aligned-window geometry): 8-row last stage without the star-only parts
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C5 --stencil random3d:1:0 --ocs ST_TB_BM_RT_PR --steps 4 --top 20 \
  --grid '{"bx":[64],"by":[4,8],"vx":[2],"merge":[4,8],"pr_stages":[4],"tb_steps":[2],"env:MIDR":[2,3]}' \
  > gpurun_out/tune_c5r1_m8b.log 2>&1
