#!/bin/bash
# final tree after removing the persistent TB-RT schedule: GPU suite + smoke, C5 / C2 / C1 / N2 bench lines
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/gputest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
python bench.py > gpurun_out/r02j_bench_C5.json 2> gpurun_out/r02j_bench_C5.err
python bench.py --config C2 > gpurun_out/r02j_bench_C2.json 2> gpurun_out/r02j_bench_C2.err
python bench.py --config C1 > gpurun_out/r02j_bench_C1.json 2> gpurun_out/r02j_bench_C1.err
python bench.py --config N2 > gpurun_out/r02j_bench_N2.json 2> gpurun_out/r02j_bench_N2.err
