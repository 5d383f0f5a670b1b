set -u
mkdir -p gpurun_out
T="timeout 600"
for st in random2d:1:0 random2d:3:8 random2d:4:12; do
$T python scripts/dev_tune.py --cfg N2 --stencil $st --ocs ST_RT_PR --steps 4 --top 8 --grid \
  '{"bx":[128,256],"vx":[2],"pr_stages":[2,3],"stream_chunk":[64,96,128,160,200,256,320,512]}' > gpurun_out/chunk2_$st.log 2>&1
done
for st in random2d:1:0 random2d:3:8 random2d:4:12; do echo == $st; grep -A8 "=== top" gpurun_out/chunk2_$st.log; done
