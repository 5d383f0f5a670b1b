set -u
mkdir -p gpurun_out
T="timeout 900"
$T python scripts/dev_tune.py --cfg N2 --stencil random2d:3:8 --ocs ST_RT_PR --steps 4 --grid \
  '{"env:NO_TMA":[0,1],"bx":[64,128,256],"vx":[2],"pr_stages":[2,4,8],"stream_chunk":[0,512]}' > gpurun_out/tune_n2_st.log 2>&1
$T python scripts/dev_tune.py --cfg N2 --stencil random2d:3:8 --ocs BM,TB_BM --steps 4 --grid \
  '{"bx":[32,64,128],"by":[4,8,16],"merge":[2,4,8],"tb_steps":[2]}' > gpurun_out/tune_n2_bm.log 2>&1
tail -n 12 gpurun_out/tune_n2_st.log gpurun_out/tune_n2_bm.log
