set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "tb_rt or run_host" > gpurun_out/chk_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/chk_pytest.log
timeout 900 python bench.py --no-cpu > gpurun_out/chk_c2.json 2> gpurun_out/chk_c2.err; echo "bench rc=$?"
python -c "import json;d=json.loads(open('gpurun_out/chk_c2.json').read().strip().splitlines()[-1]);print(d['value'], d['roofline']['frac'], d['e2e'])"
