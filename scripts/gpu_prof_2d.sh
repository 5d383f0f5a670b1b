set -u
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_stream -s 2 -c 1 -o gpurun_out/prof_n2r3 -f \
  python scripts/dev_tune.py --cfg N2 --stencil random2d:3:8 --ocs ST_RT_PR --steps 4 --grid '{"bx":[128],"vx":[2],"pr_stages":[3]}' > gpurun_out/prof_n2r3.log 2>&1
