#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
T="python scripts/dev_time.py --cfg C2 --ocs ST_TB_BM_RT_PR --reps 5"
for rep in 1 2; do
  for prm in '{}' '{"pr_stages":4}' '{"pr_stages":6}' '{"pr_stages":8}'; do
    echo "== [$rep] $prm"; $T --params "$prm" 2>&1 | grep -v Warn
    echo "== [$rep] MIDR=3 $prm"; STENCIL_MIDR=3 $T --params "$prm" 2>&1 | grep -v Warn
  done
done
