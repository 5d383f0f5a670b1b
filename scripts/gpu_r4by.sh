set -u
for rep in 1 2; do
timeout 600 python scripts/dev_time.py --cfg C5 --stencil random3d:4:12 --ocs ST_BM_RT_PR --steps 1 --reps 3 --params '{"by":2}'
timeout 600 python scripts/dev_time.py --cfg C5 --stencil random3d:4:12 --ocs ST_BM_RT_PR --steps 1 --reps 3
timeout 600 python scripts/dev_time.py --cfg C5 --stencil random3d:3:8 --ocs ST_BM_RT_PR --steps 1 --reps 3 --params '{"by":2}'
timeout 600 python scripts/dev_time.py --cfg C5 --stencil random3d:3:8 --ocs ST_BM_RT_PR --steps 1 --reps 3
done
