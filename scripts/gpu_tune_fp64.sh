# parameter headroom of the FP64-bound single-step kernels (C5 r=2/3 stencils, C4 box) at 512^3
set -u
mkdir -p gpurun_out
for st in random3d:2:4 random3d:3:8 box125; do
  timeout 900 python scripts/dev_tune.py --cfg C2 --stencil $st --ocs ST_BM_RT_PR --steps 4 --top 8 --grid \
    '{"bx":[64,128],"by":[1,2,4],"merge":[2,4],"vx":[2],"pr_stages":[2,3]}' > gpurun_out/tunefp_$st.log 2>&1
  echo "== $st"; tail -9 gpurun_out/tunefp_$st.log
done
