set -u
mkdir -p gpurun_out
timeout 600 python bench.py --config C2 --slab --transport p2p --steps 10 --no-e2e --no-cpu > gpurun_out/bench_c2_slab_p2p.json 2> gpurun_out/bench_c2_slab_p2p.err
timeout 600 python bench.py --config C2 --slab --steps 10 --no-e2e --no-cpu > gpurun_out/bench_c2_slab_nccl.json 2> gpurun_out/bench_c2_slab_nccl.err
tail -n 2 gpurun_out/bench_c2_slab_p2p.err
