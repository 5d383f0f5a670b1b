set -u
mkdir -p gpurun_out
for st in random2d:3:8 random2d:4:12 random2d:2:4; do
timeout 900 python scripts/dev_tune.py --cfg N2 --stencil $st --ocs ST_BM_RT_PR,ST_RT_PR,ST_PR --steps 4 --top 6 --grid \
  '{"bx":[128,256],"merge":[1],"vx":[2,4],"pr_stages":[2,3,4,8],"stream_chunk":[0,256,1024]}' > gpurun_out/tune2db_$st.log 2>&1
echo "== $st"; tail -7 gpurun_out/tune2db_$st.log
done
