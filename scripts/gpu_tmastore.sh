set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tma_store" > gpurun_out/tmas_pytest.log 2>&1; echo rc=$? >> gpurun_out/tmas_pytest.log
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 4 --grid \
  '{"env:OSTAGE":[0,1],"bx":[64,128],"by":[4,8],"merge":[2,4],"vx":[2],"pr_stages":[3],"tb_steps":[2]}' \
  > gpurun_out/tune_c2_tmas.log 2>&1
tail -n 3 gpurun_out/tmas_pytest.log
