#!/bin/bash
# A/B: 2-column (16-byte vector) full-width intermediate tiles of k_tiled (STENCIL_TILED_MVX=2); parity forced on
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
STENCIL_TILED_MVX=2 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py -m gpu -x -q \
  -k "every_oc or edge_every_oc or full_grid or 2d or label_pass" > gpurun_out/tmvx_parity.log 2>&1; echo "rc=$?" >> gpurun_out/tmvx_parity.log
for st in random2d:1:0 random2d:2:4 random2d:3:8; do
  timeout 600 python scripts/dev_tune.py --cfg N2 --stencil $st --ocs TB_BM --steps 10 --top 20 \
    --grid '{"bx":[64],"by":[8],"vx":[2],"merge":[4],"tb_steps":[2],"env:TILED_MVX":[1,2],"env:TILED_MID":[4,5]}' \
    > gpurun_out/ab_tmvx_${st//:/_}.log 2>&1
done
timeout 600 python scripts/dev_tune.py --cfg C2 --ocs TB_BM --steps 10 --top 20 \
    --grid '{"bx":[32],"by":[4],"bz":[4],"vx":[2],"merge":[2],"tb_steps":[2],"env:TILED_MVX":[1,2],"env:TILED_MID":[4,5]}' \
    > gpurun_out/ab_tmvx_c2.log 2>&1
timeout 600 python scripts/dev_tune.py --cfg C5 --stencil random3d:2:4 --ocs TB_BM --steps 2 --top 20 \
    --grid '{"bx":[32],"by":[4],"bz":[4],"vx":[2],"merge":[2],"tb_steps":[2],"env:TILED_MVX":[1,2]}' \
    > gpurun_out/ab_tmvx_c5r2.log 2>&1
