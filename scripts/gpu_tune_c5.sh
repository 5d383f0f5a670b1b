#!/bin/bash
# C5 FP64-bound stencils (orders 2..4): parameter grid of the retiming streaming OC
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for st in random3d:2:4 random3d:3:8 random3d:4:12; do
  timeout 900 python scripts/dev_tune.py --cfg C5 --stencil $st --ocs ST_BM_RT_PR,ST_CM_RT_PR --steps 2 --top 10 \
    --grid '{"bx":[64,128,256],"by":[1,2,4],"vx":[2],"merge":[2,4],"pr_stages":[2,3]}' \
    > gpurun_out/tune_c5_${st//:/_}.log 2>&1
done
