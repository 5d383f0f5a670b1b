#!/bin/bash
# re-entry check of the restored tree: build, GPU tests, smoke, C5 and C2 bench lines
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/gputest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/r02b_bench_C5.json 2> gpurun_out/r02b_bench_C5.err
timeout 600 python bench.py --config C2 > gpurun_out/r02b_bench_C2.json 2> gpurun_out/r02b_bench_C2.err
