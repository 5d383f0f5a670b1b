# A/B of the default z-chunk rule (STENCIL_CHUNK_RULE=old vs new), default settings
set -u
mkdir -p gpurun_out
L=gpurun_out/chunk4.log; : > $L
for rule in old new; do
  echo "=== rule $rule" >> $L
  export STENCIL_CHUNK_RULE=$rule
  timeout 300 python scripts/dev_time.py --cfg C2 --ocs ST,ST_PR,ST_RT_PR,ST_BM_RT_PR,ST_CM_PR,ST_BM --steps 10 --reps 3 >> $L 2>&1
  timeout 300 python scripts/dev_time.py --cfg C2 --stencil random3d:2:4 --ocs ST_BM_RT_PR,ST_CM_RT_PR,ST_RT_PR --steps 4 --reps 3 >> $L 2>&1
  timeout 300 python scripts/dev_time.py --cfg C2 --stencil random3d:3:8 --ocs ST_BM_RT_PR --steps 4 --reps 3 >> $L 2>&1
  timeout 300 python scripts/dev_time.py --cfg C4 --ocs ST_RT_PR,ST_CM_RT_PR,ST_BM_RT_PR --steps 10 --reps 3 >> $L 2>&1
  timeout 300 python scripts/dev_time.py --cfg C3 --ocs ST_BM_RT_PR,ST_CM_RT_PR,ST_RT_PR,ST_PR --steps 10 --reps 3 >> $L 2>&1
  timeout 600 python scripts/dev_time.py --cfg C5 --stencil random3d:2:4 --ocs ST_BM_RT_PR,ST_CM_RT_PR --steps 4 --reps 3 >> $L 2>&1
  timeout 600 python scripts/dev_time.py --cfg C5 --stencil random3d:3:8 --ocs ST_BM_RT_PR --steps 2 --reps 2 >> $L 2>&1
done
cat $L | awk '{print $1, $2, $3, $4, $5}'
