set -u
mkdir -p gpurun_out
B="python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_stream_tb_rt -s 3 -c 1 -o gpurun_out/prof_c2_v6 -f \
  $B --config C2 --oc ST_TB_BM_RT_PR > gpurun_out/prof_c2_v6.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2_v6.csv \
  $B --config C2 --oc ST_TB_BM_RT_PR > gpurun_out/launches_c2_v6.log 2>&1
ls -la gpurun_out | grep v6
