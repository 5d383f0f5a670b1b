set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tb_rt or every_oc or dyadic" > gpurun_out/tbrt_pytest.log 2>&1; echo rc=$? >> gpurun_out/tbrt_pytest.log
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 4 --grid \
  '{"env:MIDR":[2,3,4],"bx":[64,128],"by":[4,8],"merge":[2,4],"vx":[2],"pr_stages":[3],"tb_steps":[2]}' \
  > gpurun_out/tune_c2_midr.log 2>&1
tail -n 3 gpurun_out/tbrt_pytest.log
