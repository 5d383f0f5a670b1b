set -u
for st in random3d:2:4 random3d:3:8; do
for r in 0 64 72 80 96; do
  if [ $r = 0 ]; then unset STENCIL_MAXRREG; else export STENCIL_MAXRREG=$r; fi
  echo "== $st maxreg=$r"
  timeout 600 python scripts/dev_time.py --cfg C2 --stencil $st --ocs ST_BM_RT_PR,ST_CM_RT_PR --steps 4 --reps 3 | awk '{print $1,$2,$3,$4,$5,$10,$11}'
done
done
