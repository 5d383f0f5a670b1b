set -u
mkdir -p gpurun_out
N="ncu --set full --clock-control none --import-source on -s 2 -c 1 -f"
timeout 600 $N -k regex:k_tiled -o gpurun_out/profF_n2r1 python scripts/dev_prof_one.py N2 random2d:1:0 TB_BM '' 2 > gpurun_out/profF_n2r1.log 2>&1
timeout 600 $N -k regex:k_stream_tb_rt -o gpurun_out/profF_c5r1 python scripts/dev_prof_one.py C5 random3d:1:0 ST_TB_BM_RT_PR '' 2 > gpurun_out/profF_c5r1.log 2>&1
timeout 600 $N -k regex:k_stream -o gpurun_out/profF_c5r2 python scripts/dev_prof_one.py C5 random3d:2:4 ST_BM_RT_PR '' 1 > gpurun_out/profF_c5r2.log 2>&1
ls -la gpurun_out | grep profF
