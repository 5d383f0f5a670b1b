#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
STENCIL_WALIGN=2 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tb_rt or heat3d" > gpurun_out/gputest_walign2.log 2>&1
tail -2 gpurun_out/gputest_walign2.log
T="python scripts/dev_time.py"
for rep in 1 2; do
  for cfg in "STENCIL_WALIGN=0" "STENCIL_WALIGN=2"; do
    echo "== C2 [$rep] $cfg"; env $cfg $T --cfg C2 --ocs ST_TB_BM_RT_PR,ST_TB_CM_RT_PR --reps 5 2>&1 | grep -v Warn
    echo "== C5r1 [$rep] $cfg"; env $cfg $T --cfg C5 --stencil random3d:1:0 --ocs ST_TB_BM_RT_PR --steps 4 --reps 3 2>&1 | grep -v Warn
  done
done
bash scripts/gpu_prof_c2.sh r02_c2_tbrt_walign2 STENCIL_WALIGN=2
