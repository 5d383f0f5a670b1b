#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
T="python scripts/dev_time.py --cfg C2 --reps 5"
$T --ocs ST_TB_BM_RT_PR,ST_TB_CM_RT_PR,ST_TB_RT_PR,ST_TB_BM_RT 2>&1 | grep -v Warn
for prm in '{"tb_steps":3,"by":4}' '{"tb_steps":3,"by":4,"merge":2}' '{"tb_steps":3,"by":2}' '{"tb_steps":3,"bx":32,"by":8}' '{"tb_steps":4,"by":2}' '{"by":16,"merge":2}' '{"bx":128,"by":4}'; do
  echo "-- $prm"; $T --ocs ST_TB_BM_RT_PR --params "$prm" 2>&1 | grep -v Warn
done
python scripts/dev_time.py --cfg C5 --stencil random3d:1:0 --ocs ST_TB_BM_RT_PR,ST_TB_CM_RT_PR --steps 4 --reps 3
