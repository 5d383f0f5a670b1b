#!/bin/bash
# balanced z-chunks: C3's auto chunk is 512 of 760 planes (two chunks of 512 + 248)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C3 --ocs ST_CM_RT_PR,ST_BM_RT_PR --steps 4 --top 30 \
  --grid '{"bx":[128],"by":[4],"vx":[4],"merge":[2],"pr_stages":[3],"stream_chunk":[0,512,380,254,190,128,760]}' \
  > gpurun_out/tune_chunk_c3.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_RT_PR,ST_TB_BM_RT_PR --steps 10 --top 30 \
  --grid '{"stream_chunk":[0,255,170,128]}' > gpurun_out/tune_chunk_c2.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C4 --ocs ST_CM_RT_PR --steps 4 --top 30 \
  --grid '{"stream_chunk":[0,255,170,128]}' > gpurun_out/tune_chunk_c4.log 2>&1
