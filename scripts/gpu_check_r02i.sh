#!/bin/bash
# final tree: GPU suite + smoke, C5 / C2 bench lines, C1 with and without CUDA-graph replay
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/gputest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
python bench.py > gpurun_out/r02i_bench_C5.json 2> gpurun_out/r02i_bench_C5.err
python bench.py --config C2 --no-cpu > gpurun_out/r02i_bench_C2.json 2> gpurun_out/r02i_bench_C2.err
for gr in 0 1 0 1; do
  STENCIL_GRAPHS=$gr python bench.py --config C1 --no-cpu > gpurun_out/r02i_bench_C1_g$gr.json 2>> gpurun_out/r02i_bench_C1.err
  python -c "import json; d=json.load(open('gpurun_out/r02i_bench_C1_g$gr.json')); print('graphs=$gr', d['value'], d['e2e']['value'], d['e2e'].get('ms_per_step'))" >> gpurun_out/c1_graphs.txt
done
