set -u
mkdir -p gpurun_out
timeout 1500 python scripts/dev_tune.py --cfg C3 --ocs ST_BM_RT_PR,ST_RT_PR --steps 4 --top 14 --grid \
  '{"bx":[64,128],"by":[2,4,8,16],"merge":[1,2],"vx":[4],"pr_stages":[3]}' > gpurun_out/tunec3b.log 2>&1
tail -15 gpurun_out/tunec3b.log
timeout 900 python scripts/dev_tune.py --cfg C4 --ocs ST_RT_PR,ST_CM_RT_PR --steps 4 --top 8 --grid \
  '{"bx":[64,128],"by":[2,4,8],"merge":[1,2],"vx":[2],"pr_stages":[2,3]}' > gpurun_out/tunec4b.log 2>&1
tail -9 gpurun_out/tunec4b.log
