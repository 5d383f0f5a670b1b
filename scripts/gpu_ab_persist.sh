#!/bin/bash
# persistent k_stream_tb_rt schedule + CUDA graph replay: parity, C2 A/B, C2 bench
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "persistent or graph_replay or tb_rt or full_grid" \
  > gpurun_out/persist_parity.log 2>&1; echo "rc=$?" >> gpurun_out/persist_parity.log
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR,ST_TB_CM_RT_PR,ST_TB_RT_PR --steps 10 --top 16 \
  --grid '{"env:TBRT_PERSIST":[0,1]}' > gpurun_out/ab_persist_c2.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 10 --top 16 \
  --grid '{"env:TBRT_PERSIST":[1,0]}' > gpurun_out/ab_persist_c2_rep.log 2>&1
timeout 600 python bench.py --config C2 --no-cpu > gpurun_out/r02h_bench_C2.json 2> gpurun_out/r02h_bench_C2.err
timeout 600 python bench.py --config C1 --no-cpu > gpurun_out/r02h_bench_C1.json 2> gpurun_out/r02h_bench_C1.err
