set -u
for rep in 1 2; do
timeout 600 python scripts/dev_time.py --cfg C3 --ocs ST_BM_RT_PR,ST_CM_RT_PR,ST_RT_PR,ST_PR --steps 10 --reps 3
timeout 600 python scripts/dev_time.py --cfg C2 --stencil random3d:3:8 --ocs ST_BM_RT_PR,ST_RT_PR --steps 4 --reps 3
timeout 600 python scripts/dev_time.py --cfg C2 --stencil random3d:4:12 --ocs ST_BM_RT_PR --steps 2 --reps 3
done
