#!/bin/bash
# C2 TB-RT: smaller tiles with 2 CTAs per SM (MINB 2) vs the 1-CTA default; N2 order-2 TB grids
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg C2 --ocs ST_TB_BM_RT_PR --steps 10 --top 12 \
  --grid '{"bx":[64,128],"by":[4,8],"vx":[2],"merge":[2,4],"pr_stages":[3,4],"tb_steps":[2],"env:MINB":[1,2]}' \
  > gpurun_out/tune_c2_tbrt.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg N2 --stencil random2d:2:4 --ocs TB_BM,TB_CM --steps 10 --top 12 \
  --grid '{"bx":[32,64,128,256],"by":[2,4,8],"vx":[2],"merge":[2,4,8],"tb_steps":[2,4]}' \
  > gpurun_out/tune_n2_r2_tb.log 2>&1
timeout 900 python scripts/dev_tune.py --cfg N2 --stencil random2d:2:4 --ocs ST_TB_BM_RT_PR,ST_TB_RT_PR,ST_BM_RT_PR --steps 10 --top 12 \
  --grid '{"bx":[128,256],"by":[1,2,4],"vx":[2],"merge":[2],"pr_stages":[3,4],"tb_steps":[2,4]}' \
  > gpurun_out/tune_n2_r2_st.log 2>&1
# fp64 coefficients from the constant bank (LDCU.128 into uniform registers) vs UMOV-materialised immediates
for st in random3d:2:4 random3d:3:8 random3d:4:12; do
  timeout 600 python scripts/dev_tune.py --cfg C5 --stencil $st --ocs ST_BM_RT_PR,ST_CM_RT_PR --steps 2 --top 8 \
    --grid '{"bx":[128],"by":[1,2],"vx":[2],"merge":[2,4],"pr_stages":[2,3],"env:CBANK":[0,1]}' \
    > gpurun_out/tune_cbank_${st//:/_}.log 2>&1
done
timeout 600 python scripts/dev_tune.py --cfg C4 --ocs ST_CM_RT_PR,ST_RT_PR --steps 4 --top 8 \
    --grid '{"bx":[128],"by":[2],"vx":[2],"merge":[2],"pr_stages":[3],"env:CBANK":[0,1]}' > gpurun_out/tune_cbank_c4.log 2>&1
