#!/bin/bash
# round-2 final bench lines of every workload (un-profiled), final tree
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python bench.py > gpurun_out/r02m_bench_C5.json 2> gpurun_out/r02m_bench_C5.err
python bench.py --config C2 > gpurun_out/r02m_bench_C2.json 2> gpurun_out/r02m_bench_C2.err
python bench.py --config N2 > gpurun_out/r02m_bench_N2.json 2> gpurun_out/r02m_bench_N2.err
python bench.py --config C3 > gpurun_out/r02m_bench_C3.json 2> gpurun_out/r02m_bench_C3.err
python bench.py --config C4 > gpurun_out/r02m_bench_C4.json 2> gpurun_out/r02m_bench_C4.err
python bench.py --config C1 > gpurun_out/r02m_bench_C1.json 2> gpurun_out/r02m_bench_C1.err
python bench.py --impl reference > gpurun_out/r02m_bench_C5_reference.json 2> gpurun_out/r02m_bench_C5_reference.err
ncu --set full --import-source on --clock-control none -k regex:k_stream_tb_rt -s 2 -c 1 -o gpurun_out/r02m_c2_tbrt_full \
    python scripts/dev_prof_one.py C2 heat3d ST_TB_BM_RT_PR "" 2 > gpurun_out/r02m_c2_full.log 2>&1
