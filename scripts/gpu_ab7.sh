# k_tiled: intermediate steps unrolled (constant extents) + register tiles (TILED_MID): parity + A/B
set -u
mkdir -p gpurun_out
L=gpurun_out/ab7.log; : > $L
STENCIL_TILED_MID=4 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "every_oc or dyadic or run_host" > gpurun_out/ab7_pytest.log 2>&1; echo "pytest(tiled_mid 4) rc=$?" >> $L
tail -2 gpurun_out/ab7_pytest.log >> $L
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "every_oc" > gpurun_out/ab7_pytest0.log 2>&1; echo "pytest(default) rc=$?" >> $L
for rep in 1 2; do
for t in 0 2 4 8; do
  echo "== TILED_MID=$t" >> $L
  STENCIL_TILED_MID=$t timeout 300 python scripts/dev_time.py --cfg N2 --stencil random2d:1:0 --ocs TB_BM,TB --steps 10 --reps 3 --params '{"bx":64}' >> $L 2>&1
  STENCIL_TILED_MID=$t timeout 300 python scripts/dev_time.py --cfg N2 --stencil random2d:2:4 --ocs TB_BM --steps 10 --reps 3 --params '{"bx":64}' >> $L 2>&1
  STENCIL_TILED_MID=$t timeout 300 python scripts/dev_time.py --cfg C2 --ocs TB,TB_BM --steps 10 --reps 3 >> $L 2>&1
done
done
cat $L | awk '{print $1,$2,$3,$4,$5}'
