# A/B: baked strides and the k_stream_tb_rt register split (dev_time, same box)
set -u
mkdir -p gpurun_out
L=gpurun_out/ab1.log; : > $L
P='{"bx":64,"by":8,"vx":2,"merge":4,"tb_steps":2,"pr_stages":3}'
for rep in 1 2; do
for v in "STENCIL_NO_BAKE=1" "STENCIL_NO_BAKE=0" "STENCIL_REGSPLIT=64,88" "STENCIL_REGSPLIT=56,112"; do
  echo "== C2 TBRT $v" >> $L
  env $v timeout 300 python scripts/dev_time.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 10 --reps 5 --params "$P" >> $L 2>&1
done
done
for v in "STENCIL_NO_BAKE=1" "STENCIL_NO_BAKE=0"; do
  echo "== C2 ST $v" >> $L
  env $v timeout 300 python scripts/dev_time.py --cfg C2 --ocs ST_RT_PR,ST_BM_RT_PR,ST_PR --steps 10 --reps 5 >> $L 2>&1
  echo "== C3 $v" >> $L
  env $v timeout 300 python scripts/dev_time.py --cfg C3 --ocs ST_BM_RT_PR,ST_RT_PR --steps 10 --reps 5 >> $L 2>&1
  echo "== C4 $v" >> $L
  env $v timeout 300 python scripts/dev_time.py --cfg C4 --ocs ST_RT_PR --steps 10 --reps 5 >> $L 2>&1
done
cat $L
