set -u
mkdir -p gpurun_out
timeout 1200 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 4 --grid \
  '{"env:MID_ROWS":[2,3,4],"bx":[64,128],"by":[8,16],"merge":[1,2,4],"vx":[2],"pr_stages":[3],"tb_steps":[2]}' \
  > gpurun_out/tune_c2_mi.log 2>&1
