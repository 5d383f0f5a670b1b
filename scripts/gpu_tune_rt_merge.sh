#!/bin/bash
# RT streaming OCs: tile height / merge factor across the 3-D workloads (default by 2, merge 2)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for st in random3d:1:0 random3d:2:4 random3d:3:8 random3d:4:12; do
  timeout 900 python scripts/dev_tune.py --cfg C5 --stencil $st --ocs ST_BM_RT_PR,ST_CM_RT_PR --steps 2 --top 8 \
    --grid '{"by":[1,2],"merge":[2,4]}' > gpurun_out/tune_rtm_c5_${st//:/_}.log 2>&1
done
for cfg in C2 C3 C4; do
  timeout 900 python scripts/dev_tune.py --cfg $cfg --ocs ST_BM_RT_PR,ST_CM_RT_PR --steps 4 --top 8 \
    --grid '{"by":[1,2,4],"merge":[2,4]}' > gpurun_out/tune_rtm_$cfg.log 2>&1
done
