set -u
for st in random3d:1:0 random3d:1:1 random3d:1:2 heat3d; do
for pr in 3 4; do
echo "== $st pr=$pr"
timeout 300 python scripts/dev_time.py --cfg C2 --stencil $st --ocs ST_TB_BM_RT_PR,ST_TB_CM_RT_PR --steps 10 --reps 5 --params "{\"pr_stages\":$pr}" | awk '{print $1,$2,$3,$4,$5}'
done
done
