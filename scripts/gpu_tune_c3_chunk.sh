# C3: concurrent-streaming chunk length (stream_chunk) x PR depth around the default setting
set -u
mkdir -p gpurun_out
timeout 1200 python scripts/dev_tune.py --cfg C3 --ocs ST_CM_RT_PR,ST_BM_RT_PR --steps 4 --top 16 --grid \
  '{"bx":[128],"by":[4,8],"merge":[2],"vx":[4],"stream_chunk":[0,128,256,512],"pr_stages":[3,4]}' > gpurun_out/tunec3chunk.log 2>&1
tail -17 gpurun_out/tunec3chunk.log
