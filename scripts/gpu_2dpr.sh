set -u
for rep in 1 2; do
for st in random2d:3:8 random2d:4:12; do
for pr in 3 4 6; do
  echo "== $st pr=$pr"
  timeout 300 python scripts/dev_time.py --cfg N2 --stencil $st --ocs ST_BM_RT_PR,ST_RT_PR,ST_CM_RT_PR --steps 10 --reps 3 --params "{\"pr_stages\":$pr}" | awk '{print $1,$2,$3,$4,$5}'
done
done
done
