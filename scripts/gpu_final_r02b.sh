#!/bin/bash
# round-2 (re-entry) bench lines (un-profiled) and ncu evidence of the final kernels
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python bench.py > gpurun_out/r02c_bench_C5.json 2> gpurun_out/r02c_bench_C5.err
python bench.py --config C2 > gpurun_out/r02c_bench_C2.json 2> gpurun_out/r02c_bench_C2.err
python bench.py --config N2 > gpurun_out/r02c_bench_N2.json 2> gpurun_out/r02c_bench_N2.err
python bench.py --config C1 > gpurun_out/r02c_bench_C1.json 2> gpurun_out/r02c_bench_C1.err
python bench.py --config C3 --no-e2e > gpurun_out/r02c_bench_C3.json 2> gpurun_out/r02c_bench_C3.err
python bench.py --config C4 --no-e2e > gpurun_out/r02c_bench_C4.json 2> gpurun_out/r02c_bench_C4.err
python bench.py --impl reference > gpurun_out/r02c_bench_C5_reference.json 2> gpurun_out/r02c_bench_C5_reference.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02c_c5_launches.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/r02c_c5_launches_bench.log 2>&1
echo "launch list rc=$?"
for spec in "c5_r4 C5 random3d:4:12 ST_BM_RT_PR k_stream" "c5_r3 C5 random3d:3:8 ST_BM_RT_PR k_stream" \
            "c5_r2 C5 random3d:2:4 ST_BM_RT_PR k_stream" "c5_r1 C5 random3d:1:0 ST_TB_BM_RT_PR k_stream_tb_rt" \
            "c2 C2 heat3d ST_TB_BM_RT_PR k_stream_tb_rt" "n2_r2 N2 random2d:2:4 TB_BM k_tiled"; do
  set -- $spec
  ncu --set full --import-source on --clock-control none -k regex:$5 -s 2 -c 1 -o gpurun_out/r02c_$1_full \
      python scripts/dev_prof_one.py $2 $3 $4 > gpurun_out/r02c_$1_full.log 2>&1
  echo "$1 rc=$?"
done
