#!/bin/bash
# 8-row last-stage TB-RT setting for radius-1 in-plane stars (stencil_plan_create): parity, C2 A/B, bench
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/gputest.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR,ST_TB_BM_RT --steps 10 --top 16 \
  --grid '{"env:NO_M8":[0,1]}' > gpurun_out/ab_m8_c2.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 10 --top 16 \
  --grid '{"env:NO_M8":[1,0]}' > gpurun_out/ab_m8_c2_rep.log 2>&1
python bench.py --config C2 > gpurun_out/r02k_bench_C2.json 2> gpurun_out/r02k_bench_C2.err
python bench.py > gpurun_out/r02k_bench_C5.json 2> gpurun_out/r02k_bench_C5.err
