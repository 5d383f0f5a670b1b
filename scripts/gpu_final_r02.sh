#!/bin/bash
# round-2 bench lines (un-profiled) and ncu evidence
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python bench.py > gpurun_out/r02_bench_C5.json 2> gpurun_out/r02_bench_C5.err
python bench.py --config C2 > gpurun_out/r02_bench_C2.json 2> gpurun_out/r02_bench_C2.err
python bench.py --config N2 > gpurun_out/r02_bench_N2.json 2> gpurun_out/r02_bench_N2.err
python bench.py --config C1 > gpurun_out/r02_bench_C1.json 2> gpurun_out/r02_bench_C1.err
python bench.py --impl reference > gpurun_out/r02_bench_C5_reference.json 2> gpurun_out/r02_bench_C5_reference.err
bash scripts/gpu_prof_r02.sh > gpurun_out/r02_prof.log 2>&1
