#!/bin/bash
# A/B: full-width 1 x MT intermediate tiles of k_tiled (STENCIL_TILED_FULL, MT = STENCIL_TILED_MID) on N2;
# parity with them forced on; full GPU suite + C2 bench for the 32-bit frame copy
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for st in random2d:1:0 random2d:2:4; do
  timeout 600 python scripts/dev_tune.py --cfg N2 --stencil $st --ocs TB_BM --steps 10 --top 20 \
    --grid '{"bx":[64],"by":[4,8],"vx":[2],"merge":[4],"tb_steps":[2],"env:TILED_FULL":[0,1],"env:TILED_MID":[4,5]}' \
    > gpurun_out/ab_tfull_${st//:/_}.log 2>&1
done
timeout 600 python scripts/dev_tune.py --cfg C2 --ocs TB_BM,TB --steps 10 --top 20 \
    --grid '{"bx":[32],"by":[4],"bz":[4],"vx":[2],"merge":[2],"tb_steps":[2],"env:TILED_FULL":[0,1],"env:TILED_MID":[4,5]}' \
    > gpurun_out/ab_tfull_c2.log 2>&1
STENCIL_TILED_FULL=1 STENCIL_TILED_MID=5 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py -m gpu -x -q \
  -k "every_oc or edge_every_oc or full_grid or 2d or label_pass" > gpurun_out/tfull_parity.log 2>&1; echo "rc=$?" >> gpurun_out/tfull_parity.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/gputest.log
python bench.py --config C2 --no-cpu > gpurun_out/r02e_bench_C2.json 2> gpurun_out/r02e_bench_C2.err
