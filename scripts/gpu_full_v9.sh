set -u
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/ -x -q -m gpu > gpurun_out/v9_pytest.log 2>&1; echo "pytest rc=$?" > gpurun_out/v9.log
tail -3 gpurun_out/v9_pytest.log >> gpurun_out/v9.log
for cfg in C2 C3 C4 N2 C1 C5; do
  timeout 1200 python bench.py --config $cfg > gpurun_out/v9_bench_$cfg.json 2> gpurun_out/v9_bench_$cfg.err
  echo "$cfg rc=$?" >> gpurun_out/v9.log
done
cat gpurun_out/v9.log
