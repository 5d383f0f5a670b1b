set -u
mkdir -p gpurun_out
L=gpurun_out/ab4.log; : > $L
timeout 1200 python -m pytest tests/ -x -q -m gpu > gpurun_out/ab4_pytest.log 2>&1; echo "pytest rc=$?" >> $L
tail -3 gpurun_out/ab4_pytest.log >> $L
P='{"bx":64,"by":8,"vx":2,"merge":4,"tb_steps":2,"pr_stages":3}'
for v in "STENCIL_X=0" "STENCIL_XSHIFT=0"; do
  for st in random3d:1:0 random3d:1:1 heat3d; do
    echo "== $st $v" >> $L
    env $v timeout 300 python scripts/dev_time.py --cfg C2 --stencil $st --ocs ST_TB_BM_RT_PR --steps 10 --reps 5 --params "$P" >> $L 2>&1
  done
done
timeout 900 python bench.py --config C5 > gpurun_out/ab4_c5.json 2>gpurun_out/ab4_c5.err; echo "c5 rc=$?" >> $L
cat $L
