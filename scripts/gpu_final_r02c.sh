#!/bin/bash
# round-2 final: GPU suite + smoke, bench lines of every workload (un-profiled), C5 launch list,
# ncu --set full of the round-2 k_tiled TB kernels at 2 fused steps
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/gputest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
python bench.py > gpurun_out/r02g_bench_C5.json 2> gpurun_out/r02g_bench_C5.err
python bench.py --config C2 > gpurun_out/r02g_bench_C2.json 2> gpurun_out/r02g_bench_C2.err
python bench.py --config N2 > gpurun_out/r02g_bench_N2.json 2> gpurun_out/r02g_bench_N2.err
python bench.py --config C1 > gpurun_out/r02g_bench_C1.json 2> gpurun_out/r02g_bench_C1.err
python bench.py --config C3 > gpurun_out/r02g_bench_C3.json 2> gpurun_out/r02g_bench_C3.err
python bench.py --config C4 > gpurun_out/r02g_bench_C4.json 2> gpurun_out/r02g_bench_C4.err
python bench.py --impl reference > gpurun_out/r02g_bench_C5_reference.json 2> gpurun_out/r02g_bench_C5_reference.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02g_c5_launches.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/r02g_c5_launches_bench.log 2>&1
echo "launch list rc=$?"
for spec in "n2_r2 N2 random2d:2:4 TB_BM k_tiled" "c2_tb C2 heat3d TB_BM k_tiled" "n2_r1 N2 random2d:1:0 TB_BM k_tiled"; do
  set -- $spec
  ncu --set full --import-source on --clock-control none -k regex:$5 -s 2 -c 1 -o gpurun_out/r02g_$1_full \
      python scripts/dev_prof_one.py $2 $3 $4 "" 2 > gpurun_out/r02g_$1_full.log 2>&1
  echo "$1 rc=$?"
done
