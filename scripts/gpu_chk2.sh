set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "run_host or xshift_remainder" > gpurun_out/chk2_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/chk2_pytest.log
timeout 900 python bench.py --config N2 --no-cpu > gpurun_out/chk2_n2.json 2> gpurun_out/chk2_n2.err; echo "bench rc=$?"
python -c "import json;d=json.loads(open('gpurun_out/chk2_n2.json').read().strip().splitlines()[-1]);print(d['value'], d['e2e'])"
