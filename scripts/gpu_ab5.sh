# even/odd-split last intermediate ring (SPLITMID): parity + A/B
set -u
mkdir -p gpurun_out
L=gpurun_out/ab5.log; : > $L
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "tb_rt or every_oc or dyadic" > gpurun_out/ab5_pytest.log 2>&1; echo "pytest rc=$?" >> $L
tail -3 gpurun_out/ab5_pytest.log >> $L
P='{"bx":64,"by":8,"vx":2,"merge":4,"tb_steps":2,"pr_stages":3}'
for rep in 1 2; do
for v in "STENCIL_SPLITMID=1" "STENCIL_SPLITMID=0"; do
  echo "== C2 TBRT $v" >> $L
  env $v timeout 300 python scripts/dev_time.py --cfg C2 --ocs ST_TB_BM_RT_PR,ST_TB_CM_RT_PR,ST_TB_RT_PR --steps 10 --reps 5 --params "$P" >> $L 2>&1
done
done
cat $L
