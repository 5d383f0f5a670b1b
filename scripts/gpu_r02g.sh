#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 120 python scripts/sanitize_case.py p2p 2>&1 | grep -v Warn | tail -1; echo "plain p2p rc=$?"
CASES="tbrt_cpasync p2p" TOOLS="racecheck memcheck synccheck" bash scripts/gpu_sanitize.sh > /dev/null 2>&1
cat gpurun_out/sanitize_summary.txt
timeout 900 python -m pytest tests/test_gpu_edge.py tests/test_gpu_parity.py tests/test_p2p.py -m gpu -q -x -k "tb_rt or asym or unaligned or p2p or heat3d" > gpurun_out/gputest_g.log 2>&1; tail -2 gpurun_out/gputest_g.log
python scripts/dev_time.py --cfg C2 --ocs ST_TB_BM_RT_PR,ST_TB_CM_RT_PR --reps 5 2>&1 | grep -v Warn
python scripts/dev_time.py --cfg C2 --ocs ST_TB_BM_RT_PR,ST_TB_CM_RT_PR --reps 5 2>&1 | grep -v Warn
