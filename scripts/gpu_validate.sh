# Full GPU validation: parity tests, smoke, default bench (N=1), launch list
set -u
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/val_gpu.txt 2>&1
timeout 1500 python -m pytest tests/ -x -q -m gpu > gpurun_out/val_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/val.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/val_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/val.log
timeout 900 python bench.py > gpurun_out/val_bench.json 2> gpurun_out/val_bench.err; echo "bench rc=$?" >> gpurun_out/val.log
cat gpurun_out/val.log; tail -3 gpurun_out/val_pytest.log; cat gpurun_out/val_bench.json | head -c 600
