#!/bin/bash
# Dev: parameter grids for the dominant kernels (run on the GPU box via gpurun).
set -u
mkdir -p gpurun_out
T="timeout 600"
$T python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 4 --grid \
  '{"bx":[64,128],"by":[4,8],"merge":[2,4],"vx":[2],"pr_stages":[3,4,6,8],"stream_chunk":[0,64,128],"tb_steps":[2]}' \
  > gpurun_out/tune_c2_tb2.log 2>&1
$T python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR,ST_TB_RT_PR --steps 4 --grid \
  '{"bx":[32,64],"by":[4,8],"merge":[1,2],"vx":[2],"pr_stages":[4,6],"stream_chunk":[0,64],"tb_steps":[4]}' \
  > gpurun_out/tune_c2_tb4.log 2>&1
$T python scripts/dev_tune.py --cfg C3 --ocs ST_BM_RT_PR --steps 4 --grid \
  '{"bx":[128,256],"by":[1,2,4],"merge":[2],"vx":[4],"pr_stages":[3,4],"stream_chunk":[0,128,256]}' \
  > gpurun_out/tune_c3_bm.log 2>&1
$T python scripts/dev_tune.py --cfg C3 --ocs ST_RT_PR --steps 4 --grid \
  '{"bx":[128,256],"by":[2,4,8],"vx":[4],"pr_stages":[3,4],"stream_chunk":[0,128,256]}' \
  > gpurun_out/tune_c3_rt.log 2>&1
tail -4 gpurun_out/tune_*.log
