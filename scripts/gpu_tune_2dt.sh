set -u
for st in random2d:1:0 random2d:2:4; do
timeout 600 python scripts/dev_tune.py --cfg N2 --stencil $st --ocs TB_BM --steps 10 --top 5 --grid \
  '{"bx":[32,64,128],"by":[2,4,8],"merge":[2,4],"vx":[2],"tb_steps":[2]}' 2>&1 | tail -6
timeout 300 python scripts/dev_time.py --cfg N2 --stencil $st --ocs TB_BM,TB,TB_CM --steps 10 --reps 3 | awk '{print $1,$2,$3,$4,$5}'
done
