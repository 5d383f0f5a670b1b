# parity (all GPU tests) + A/B of the automatic register split + default bench
set -u
mkdir -p gpurun_out
L=gpurun_out/ab2.log; : > $L
timeout 900 python -m pytest tests/ -x -q -m gpu > gpurun_out/ab2_pytest.log 2>&1; echo "pytest rc=$?" >> $L
tail -3 gpurun_out/ab2_pytest.log >> $L
P='{"bx":64,"by":8,"vx":2,"merge":4,"tb_steps":2,"pr_stages":3}'
for rep in 1 2; do
for v in "STENCIL_X=0" "STENCIL_REGSPLIT=0,0"; do
  echo "== C2 TBRT $v" >> $L
  env $v timeout 300 python scripts/dev_time.py --cfg C2 --ocs ST_TB_BM_RT_PR,ST_TB_CM_RT_PR --steps 10 --reps 5 --params "$P" >> $L 2>&1
done
done
timeout 900 python bench.py > gpurun_out/ab2_bench.json 2> gpurun_out/ab2_bench.err; echo "bench rc=$?" >> $L
cat $L; head -c 400 gpurun_out/ab2_bench.json
