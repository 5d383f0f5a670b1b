#!/bin/bash
# new k_tiled defaults (full-width 1 x 5 intermediate tiles, 2-D TB 64 x 32): GPU suite, N2 bench;
# N2 order-2 tile heights / MT 7; C2 FULLW with the corrected split pitch
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/gputest.log
python bench.py --config N2 --no-cpu > gpurun_out/r02f_bench_N2.json 2> gpurun_out/r02f_bench_N2.err
timeout 600 python scripts/dev_tune.py --cfg N2 --stencil random2d:2:4 --ocs TB_BM --steps 10 --top 20 \
    --grid '{"bx":[64,128],"by":[8,16],"vx":[2],"merge":[4],"tb_steps":[2],"env:TILED_MID":[5,7]}' > gpurun_out/ab_n2r2_mt.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 10 --top 16 \
  --grid '{"bx":[64],"by":[8],"vx":[2],"merge":[4],"pr_stages":[4],"tb_steps":[2],"env:FULLW":[0,1],"env:MID_ROWS":[4,5],"env:XSHIFT":[0]}' \
  > gpurun_out/ab_fullw_c2_v2.log 2>&1
