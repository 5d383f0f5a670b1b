#!/bin/bash
# round-2 A/B batch 1 (one box): k_stream_tb_rt hand-off switches on C2; ST_TB_RT
# without prefetch; C5 order-2/4 tile heights and chunks; N2 2-D x-merge.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
T="python scripts/dev_time.py"
for rep in 1 2; do
  for cfg in "STENCIL_ELECT=0 STENCIL_WALIGN=0" "STENCIL_ELECT=1 STENCIL_WALIGN=0" "STENCIL_ELECT=0 STENCIL_WALIGN=1" "STENCIL_ELECT=1 STENCIL_WALIGN=1"; do
    echo "== C2 [$rep] $cfg"
    env $cfg $T --cfg C2 --ocs ST_TB_BM_RT_PR,ST_TB_CM_RT_PR,ST_TB_RT_PR --reps 5 2>&1 | grep -v Warn
  done
done
echo "== C2 ST_TB_RT (no PR)"
$T --cfg C2 --ocs ST_TB_RT --reps 3
$T --cfg C2 --ocs ST_TB_RT --reps 3 --params '{"by":4}'
STENCIL_MINB=2 $T --cfg C2 --ocs ST_TB_RT --reps 3 --params '{"by":4}'
STENCIL_MINB=2 $T --cfg C2 --ocs ST_TB_RT --reps 3 --params '{"by":2}'
echo "== C5 r2 / r4"
for st in random3d:2:4 random3d:4:12; do
  for prm in '{}' '{"by":4}' '{"stream_chunk":64}' '{"by":4,"stream_chunk":64}' '{"stream_chunk":1024}'; do
    echo "-- $st $prm"; $T --cfg C5 --stencil $st --ocs ST_BM_RT_PR --steps 4 --reps 3 --params "$prm"
  done
done
echo "== N2 all OCs (x-merge)"
for st in random2d:1:0 random2d:2:4 random2d:3:8 random2d:4:12; do
  echo "-- $st"; $T --cfg N2 --stencil $st --reps 3
done
