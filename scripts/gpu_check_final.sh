#!/bin/bash
# round-end rehearsal: what the driver runs (GPU suite, smoke, default bench), on the final tree
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/gputest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
python bench.py > gpurun_out/final_bench_C5.json 2> gpurun_out/final_bench_C5.err; echo "bench rc=$?" >> gpurun_out/smoke.log
wc -l gpurun_out/final_bench_C5.json >> gpurun_out/smoke.log
