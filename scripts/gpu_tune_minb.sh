set -u
mkdir -p gpurun_out
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 4 --top 12 --grid \
  '{"env:MINB":[1,2],"bx":[32,64],"by":[4,8],"merge":[2,4],"vx":[2],"pr_stages":[2,3],"tb_steps":[2]}' > gpurun_out/tune_minb.log 2>&1
tail -13 gpurun_out/tune_minb.log
