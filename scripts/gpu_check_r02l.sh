#!/bin/bash
# after the 8-row TB-RT setting: GPU suite + smoke, C2 / C5 bench lines
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/gputest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
python bench.py --config C2 > gpurun_out/r02l_bench_C2.json 2> gpurun_out/r02l_bench_C2.err
python bench.py > gpurun_out/r02l_bench_C5.json 2> gpurun_out/r02l_bench_C5.err
