set -u
timeout 600 python scripts/dev_tune.py --cfg N2 --stencil random2d:1:0 --ocs TB_BM,TB --steps 4 --top 8 --grid \
  '{"bx":[32,64,128],"by":[4,8],"merge":[2,4],"vx":[2],"tb_steps":[2,4]}' 2>&1 | tail -9
timeout 600 python scripts/dev_tune.py --cfg N2 --stencil random2d:2:4 --ocs TB_BM --steps 4 --top 4 --grid \
  '{"bx":[32,64,128],"by":[4,8],"merge":[2,4],"vx":[2],"tb_steps":[2,4]}' 2>&1 | tail -5
timeout 600 python scripts/dev_time.py --cfg C2 --ocs TB,TB_BM,TB_CM --steps 10 --reps 3 | awk '{print $1,$2,$3,$4,$5}'
