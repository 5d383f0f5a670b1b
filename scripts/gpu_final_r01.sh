# round-1 final: GPU tests, smoke, default bench (N=1), launch list of the default bench command
set -u
mkdir -p gpurun_out
L=gpurun_out/final.log; : > $L
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv >> $L 2>&1
timeout 1500 python -m pytest tests/ -x -q -m gpu > gpurun_out/final_pytest.log 2>&1; echo "pytest rc=$?" >> $L
tail -3 gpurun_out/final_pytest.log >> $L
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.log 2>&1; echo "smoke rc=$?" >> $L
timeout 900 python bench.py > gpurun_out/final_bench_C2.json 2> gpurun_out/final_bench_C2.err; echo "bench rc=$?" >> $L
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final_ref.json 2> gpurun_out/final_ref.err; echo "ref rc=$?" >> $L
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final_launches.csv \
  python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu > gpurun_out/final_launches.log 2>&1; echo "ncu rc=$?" >> $L
cat $L; head -c 700 gpurun_out/final_bench_C2.json; echo; cat gpurun_out/final_ref.json | head -c 400
