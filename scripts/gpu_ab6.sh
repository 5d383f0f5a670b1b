# scalar-column intermediate steps (MID_VX=1): parity + A/B
set -u
mkdir -p gpurun_out
L=gpurun_out/ab6.log; : > $L
STENCIL_MID_VX=1 STENCIL_MID_ROWS=4 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "tb_rt" > gpurun_out/ab6_pytest.log 2>&1; echo "pytest(midvx1) rc=$?" >> $L
tail -3 gpurun_out/ab6_pytest.log >> $L
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "tb_rt" > gpurun_out/ab6_pytest0.log 2>&1; echo "pytest(default) rc=$?" >> $L
P='{"bx":64,"by":8,"vx":2,"merge":4,"tb_steps":2,"pr_stages":3}'
for rep in 1 2; do
for v in "STENCIL_MID_VX=0 STENCIL_MID_ROWS=2" "STENCIL_MID_VX=1 STENCIL_MID_ROWS=4" "STENCIL_MID_VX=1 STENCIL_MID_ROWS=8" "STENCIL_MID_VX=1 STENCIL_MID_ROWS=6"; do
  echo "== C2 TBRT $v" >> $L
  env $v timeout 300 python scripts/dev_time.py --cfg C2 --ocs ST_TB_BM_RT_PR,ST_TB_CM_RT_PR --steps 10 --reps 5 --params "$P" >> $L 2>&1
done
done
cat $L
