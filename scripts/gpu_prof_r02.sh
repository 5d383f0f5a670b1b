#!/bin/bash
# Round-2 evidence: (1) launch list of the default bench command (C5) under
# ncu --metrics gpu__time_duration.sum; (2) ncu --set full of the C5 dominant
# kernels (order 4 and order 1) and of C2's k_stream_tb_rt at the bench's
# default settings. Summaries: python scripts/ncu_metrics.py <rep>.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_c5_launches.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/r02_c5_launches_bench.log 2>&1
echo "launch list rc=$?"
for spec in "c5_r4 C5 random3d:4:12 ST_BM_RT_PR k_stream" "c5_r1 C5 random3d:1:0 ST_TB_BM_RT_PR k_stream_tb_rt" \
            "c5_r2 C5 random3d:2:4 ST_BM_RT_PR k_stream" "c2 C2 heat3d ST_TB_BM_RT_PR k_stream_tb_rt" \
            "n2_r2 N2 random2d:2:4 TB_BM k_tiled" "c3 C3 star25 ST_CM_RT_PR k_stream"; do
  set -- $spec
  ncu --set full --import-source on --clock-control none -k regex:$5 -s 2 -c 1 -o gpurun_out/r02_$1_full \
      python scripts/dev_prof_one.py $2 $3 $4 > gpurun_out/r02_$1_full.log 2>&1
  echo "$1 rc=$?"
done
