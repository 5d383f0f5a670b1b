set -u
mkdir -p gpurun_out
timeout 1500 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 4 --top 25 --grid \
  '{"env:MID_ROWS":[2,3,4],"pr_stages":[2,3,4,6],"tb_steps":[2,4],"merge":[2,4],"by":[8,16],"bx":[64],"vx":[2]}' \
  > gpurun_out/tune_v6.log 2>&1
tail -27 gpurun_out/tune_v6.log
