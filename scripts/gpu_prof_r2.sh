set -u
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_stream -s 2 -c 1 -o gpurun_out/prof_r2 -f \
  python scripts/dev_prof_one.py C2 random3d:2:4 ST_BM_RT_PR > gpurun_out/prof_r2.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_stream -s 2 -c 1 -o gpurun_out/prof_c3 -f \
  python scripts/dev_prof_one.py C3 star25 ST_BM_RT_PR > gpurun_out/prof_c3.log 2>&1
ls -la gpurun_out | grep prof_
