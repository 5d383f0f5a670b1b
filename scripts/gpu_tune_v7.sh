set -u
mkdir -p gpurun_out
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR,ST_TB_CM_RT_PR --steps 4 --top 12 --grid \
  '{"bx":[32,64,128],"by":[4,8,16],"merge":[4,8],"vx":[2],"pr_stages":[3],"tb_steps":[2]}' > gpurun_out/tune_v7.log 2>&1
tail -13 gpurun_out/tune_v7.log
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "run_host" > gpurun_out/v7b_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/v7b_pytest.log
for cfg in C4 C3; do timeout 900 python bench.py --config $cfg --no-cpu > gpurun_out/v7b_$cfg.json 2>/dev/null; python -c "import json;d=json.loads(open('gpurun_out/v7b_$cfg.json').read().strip().splitlines()[-1]);print('$cfg',d['value'],d['e2e'])"; done
