set -u
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/ -x -q -m gpu > gpurun_out/v11_pytest.log 2>&1; echo "pytest rc=$?" > gpurun_out/v11.log
tail -3 gpurun_out/v11_pytest.log >> gpurun_out/v11.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/v11_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/v11.log
for cfg in C2 C3 C4 N2 C1 C5; do
  timeout 1200 python bench.py --config $cfg > gpurun_out/v11_bench_$cfg.json 2> gpurun_out/v11_bench_$cfg.err
  echo "$cfg rc=$?" >> gpurun_out/v11.log
done
B="python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu"
cat gpurun_out/v11.log
