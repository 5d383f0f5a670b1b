set -u
mkdir -p gpurun_out
timeout 1500 python scripts/dev_tune.py --cfg C3 --ocs ST_BM_RT_PR,ST_CM_RT_PR --steps 4 --top 12 --grid \
  '{"bx":[64,128],"by":[1,2,4],"merge":[1,2,4],"vx":[4],"pr_stages":[2,3,4]}' > gpurun_out/tunec3.log 2>&1
tail -13 gpurun_out/tunec3.log
