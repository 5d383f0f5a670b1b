set -u
mkdir -p gpurun_out
T="timeout 600"
$T python scripts/dev_tune.py --cfg N2 --stencil random2d:3:8 --ocs ST_RT_PR --steps 4 --top 20 --grid \
  '{"bx":[128],"vx":[2],"pr_stages":[3],"stream_chunk":[16,32,48,64,96,128,200,256,512]}' > gpurun_out/chunk_n2.log 2>&1
$T python scripts/dev_tune.py --cfg N2 --stencil random2d:1:0 --ocs ST_RT_PR,ST_BM_PR --steps 4 --top 20 --grid \
  '{"bx":[128],"vx":[2],"pr_stages":[3],"stream_chunk":[32,64,128,200,512]}' > gpurun_out/chunk_n2r1.log 2>&1
$T python scripts/dev_tune.py --cfg C3 --ocs ST_BM_RT_PR --steps 4 --top 20 --grid \
  '{"bx":[128],"by":[2],"merge":[2],"vx":[4],"pr_stages":[3],"stream_chunk":[48,64,96,128,152,192,760]}' > gpurun_out/chunk_c3.log 2>&1
$T python scripts/dev_tune.py --cfg C2 --ocs ST_RT_PR --steps 4 --top 20 --grid \
  '{"bx":[128],"by":[2],"vx":[2],"pr_stages":[3],"stream_chunk":[32,64,128,170,256,510]}' > gpurun_out/chunk_c2.log 2>&1
$T python scripts/dev_tune.py --cfg C4 --ocs ST_RT_PR --steps 2 --top 20 --grid \
  '{"bx":[64,128],"by":[2,4],"vx":[2],"pr_stages":[3,4],"stream_chunk":[32,64,128,510]}' > gpurun_out/chunk_c4.log 2>&1
for f in n2 n2r1 c3 c2 c4; do echo == $f; grep -A8 "=== top" gpurun_out/chunk_$f.log; done
