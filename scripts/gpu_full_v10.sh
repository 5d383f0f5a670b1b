set -u
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/ -x -q -m gpu > gpurun_out/v10_pytest.log 2>&1; echo "pytest rc=$?" > gpurun_out/v10.log
tail -3 gpurun_out/v10_pytest.log >> gpurun_out/v10.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/v10_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/v10.log
for cfg in C2 N2; do
  timeout 1200 python bench.py --config $cfg > gpurun_out/v10_bench_$cfg.json 2> gpurun_out/v10_bench_$cfg.err
  echo "$cfg rc=$?" >> gpurun_out/v10.log
done
B="python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_stream_tb_rt -s 3 -c 1 -o gpurun_out/prof_c2_v10 -f \
  $B --config C2 --oc ST_TB_BM_RT_PR > gpurun_out/prof_c2_v10.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_tiled -s 2 -c 1 -o gpurun_out/prof_n2_v10 -f \
  python scripts/dev_prof_one.py N2 random2d:1:0 TB_BM > gpurun_out/prof_n2_v10.log 2>&1
cat gpurun_out/v10.log
