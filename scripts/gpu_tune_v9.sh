set -u
mkdir -p gpurun_out
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 10 --top 10 --grid \
  '{"bx":[64,128],"by":[4,8,16],"merge":[2,4],"vx":[2],"pr_stages":[2,3,4],"tb_steps":[2]}' > gpurun_out/tune_v9.log 2>&1
tail -11 gpurun_out/tune_v9.log
