set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "random2d or heat2d or c1 or N2" > gpurun_out/n2_pytest.log 2>&1; echo rc=$? >> gpurun_out/n2_pytest.log
timeout 900 python bench.py --config N2 > gpurun_out/bench_N2_v5.json 2> gpurun_out/bench_N2_v5.err
timeout 900 python bench.py --config C2 --no-e2e > gpurun_out/bench_C2_v5.json 2> gpurun_out/bench_C2_v5.err
tail -n 2 gpurun_out/n2_pytest.log
