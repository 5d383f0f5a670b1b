set -u
mkdir -p gpurun_out
L=gpurun_out/pipe.log; : > $L
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "run_host" > gpurun_out/pipe_pytest.log 2>&1; echo "pytest rc=$?" >> $L
tail -15 gpurun_out/pipe_pytest.log >> $L
timeout 900 python bench.py --no-cpu > gpurun_out/pipe_c2.json 2> gpurun_out/pipe_c2.err; echo "c2 rc=$?" >> $L
python -c "import json;d=json.loads(open('gpurun_out/pipe_c2.json').read().strip().splitlines()[-1]);print(d['value'],d['e2e'])" >> $L 2>&1
cat $L
