set -u
for rep in 1 2; do
for cv in -1 100; do
  export STENCIL_CARVEOUT=$cv
  echo "== carveout $cv"
  timeout 300 python scripts/dev_time.py --cfg C3 --ocs ST_CM_RT_PR,ST_BM_RT_PR --steps 10 --reps 3 | awk '{print "C3", $1,$2,$3,$4,$5}'
  timeout 300 python scripts/dev_time.py --cfg C2 --ocs ST_PR,ST_RT_PR,ST_BM,ST_TB_BM_RT_PR --steps 10 --reps 3 | awk '{print "C2", $1,$2,$3,$4,$5}'
  timeout 300 python scripts/dev_time.py --cfg C4 --ocs ST_CM_RT_PR --steps 10 --reps 3 | awk '{print "C4", $1,$2,$3,$4,$5}'
  timeout 300 python scripts/dev_time.py --cfg C2 --stencil random3d:2:4 --ocs ST_BM_RT_PR --steps 4 --reps 3 | awk '{print "r2", $1,$2,$3,$4,$5}'
  timeout 300 python scripts/dev_time.py --cfg N2 --stencil random2d:3:8 --ocs ST_BM_RT_PR,TB_BM --steps 10 --reps 3 | awk '{print "N2r3", $1,$2,$3,$4,$5}'
done
done
