#!/bin/bash
# full GPU suite + smoke on the round-2 k_tiled defaults; sanitizer subset over the new paths; N2 order-2 merge 8
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/gputest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
CASES="naive tiled_tb tiled_tb_2d tiled_tb_fp32 stream_rt tbrt_split" TOOLS="memcheck racecheck synccheck" \
  timeout 1500 bash scripts/gpu_sanitize.sh > gpurun_out/sanitize.log 2>&1
timeout 600 python scripts/dev_tune.py --cfg N2 --stencil random2d:2:4 --ocs TB_BM,TB_CM --steps 10 --top 20 \
    --grid '{"bx":[64],"by":[2,4,8],"vx":[2],"merge":[4,8],"tb_steps":[2]}' > gpurun_out/ab_n2r2_m8.log 2>&1
