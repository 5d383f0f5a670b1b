#!/bin/bash
# the slab (multi-GPU) code path at N = 1 with the final kernels: NCCL transport and fused P2P halo;
# C5 slab = per-stencil buffers (ghost depth 4 x order)
env | grep -i nccl > gpurun_out/nccl_env.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python bench.py --config C2 --slab --no-cpu > gpurun_out/r02n_bench_C2_slab.json 2> gpurun_out/r02n_bench_C2_slab.err
python bench.py --config C2 --slab --transport p2p --no-cpu --no-e2e > gpurun_out/r02n_bench_C2_p2p.json 2> gpurun_out/r02n_bench_C2_p2p.err
python bench.py --slab --no-cpu > gpurun_out/r02n_bench_C5_slab.json 2> gpurun_out/r02n_bench_C5_slab.err
python bench.py --slab --transport p2p --no-cpu --no-e2e > gpurun_out/r02n_bench_C5_p2p.json 2> gpurun_out/r02n_bench_C5_p2p.err
python bench.py --config C1 --no-cpu > gpurun_out/r02n_bench_C1.json 2> gpurun_out/r02n_bench_C1.err
