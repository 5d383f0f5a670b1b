set -u
mkdir -p gpurun_out
L=gpurun_out/dbg1.log; : > $L
for oc in ST_TB_RT ST_TB_RT_PR ST_TB_BM_RT ST_TB_BM_RT_PR ST_TB_CM_RT ST_TB_CM_RT_PR; do
  timeout 120 python scripts/dev_one_oc.py heat3d '[36,41,68]' f32 $oc >> $L 2>&1 || echo "$oc FAILED rc=$?" >> $L
done
timeout 300 compute-sanitizer --tool memcheck python scripts/dev_one_oc.py heat3d '[36,41,68]' f32 ST_TB_RT > gpurun_out/dbg1_san.log 2>&1
grep -v "^=========     Host Frame" gpurun_out/dbg1_san.log | head -60 >> $L
cat $L
