# z-chunk (stream_chunk) sweep: wave quantisation of FP-bound streaming kernels at 512^3
set -u
mkdir -p gpurun_out
for st in random3d:2:4 random3d:3:8 box125 heat3d; do
timeout 900 python scripts/dev_tune.py --cfg C2 --stencil $st --ocs ST_BM_RT_PR --steps 4 --top 20 --grid \
  '{"stream_chunk":[16,24,32,39,46,51,57,64,73,85,102,128,170,255,510]}' > gpurun_out/chunk3_$st.log 2>&1
echo "== $st"; grep "GSt/s" gpurun_out/chunk3_$st.log | head -15
done
