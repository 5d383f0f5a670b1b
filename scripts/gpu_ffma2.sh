set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "f32 or star25 or random3d or run_host" > gpurun_out/ffma2_pytest.log 2>&1; echo rc=$? >> gpurun_out/ffma2_pytest.log
timeout 900 python scripts/dev_tune.py --cfg C3 --ocs ST_BM_RT_PR,ST_RT_PR --steps 4 --grid \
  '{"env:NO_FFMA2":[0,1],"bx":[64,128],"by":[2,4,8],"merge":[1,2],"vx":[4],"pr_stages":[3],"stream_chunk":[0,128]}' \
  > gpurun_out/tune_c3_ffma2.log 2>&1
tail -n 3 gpurun_out/ffma2_pytest.log
