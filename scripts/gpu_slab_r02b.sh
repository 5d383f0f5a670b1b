#!/bin/bash
# stdout of the slab runs must be exactly one JSON line
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python bench.py --config C2 --slab --no-cpu --no-e2e --steps 5 > gpurun_out/r02o_bench_C2_slab.json 2> gpurun_out/r02o_bench_C2_slab.err
wc -l gpurun_out/r02o_bench_C2_slab.json > gpurun_out/r02o_lines.txt
