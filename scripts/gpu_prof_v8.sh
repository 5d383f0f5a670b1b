set -u
mkdir -p gpurun_out
N="ncu --set full --clock-control none --import-source on -k regex:k_stream -s 2 -c 1 -f"
timeout 600 $N -o gpurun_out/prof8_c3 python scripts/dev_prof_one.py C3 star25 ST_CM_RT_PR > gpurun_out/prof8_c3.log 2>&1
timeout 600 $N -o gpurun_out/prof8_c4 python scripts/dev_prof_one.py C4 box125 ST_CM_RT_PR '{"bx":64,"by":2,"vx":2,"merge":2,"pr_stages":2}' > gpurun_out/prof8_c4.log 2>&1
timeout 600 $N -o gpurun_out/prof8_n2 python scripts/dev_prof_one.py N2 random2d:3:8 ST_BM_RT_PR > gpurun_out/prof8_n2.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2_v8.csv \
  python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu > gpurun_out/launches_c2_v8.log 2>&1
ls -la gpurun_out | grep -E "prof8|launches_c2_v8"; tail -2 gpurun_out/prof8_*.log
