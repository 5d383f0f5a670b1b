# 2-D (N2) tiled/TB settings headroom: random2d order-1 and order-3 stencils at 8192^2
set -u
mkdir -p gpurun_out
timeout 900 python scripts/dev_tune.py --cfg N2 --stencil random2d:1:0 --ocs TB_BM,TB,TB_CM --steps 4 --top 10 --grid \
  '{"bx":[64,128,256],"by":[4,8,16,32],"merge":[1,2,4],"vx":[2],"tb_steps":[2,4]}' > gpurun_out/tune2d_r1.log 2>&1
echo "== r1"; tail -11 gpurun_out/tune2d_r1.log
timeout 900 python scripts/dev_tune.py --cfg N2 --stencil random2d:1:0 --ocs ST_TB_BM_RT_PR,ST_BM_RT_PR,ST_PR --steps 4 --top 6 --grid \
  '{"bx":[64,128,256],"merge":[1],"vx":[2],"tb_steps":[2,4],"pr_stages":[2,3,4]}' > gpurun_out/tune2d_r1s.log 2>&1
echo "== r1 streaming"; tail -7 gpurun_out/tune2d_r1s.log
timeout 900 python scripts/dev_tune.py --cfg N2 --stencil random2d:3:8 --ocs ST_BM_RT_PR,BM,TB_BM --steps 4 --top 8 --grid \
  '{"bx":[64,128,256],"by":[4,8,16],"merge":[1,2,4],"vx":[2],"pr_stages":[3],"tb_steps":[2]}' > gpurun_out/tune2d_r3.log 2>&1
echo "== r3"; tail -9 gpurun_out/tune2d_r3.log
