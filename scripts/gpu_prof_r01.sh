set -u
mkdir -p gpurun_out
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_stream -s 3 -c 1 -o gpurun_out/prof_c3 -f \
  $B --config C3 --oc ST_BM_RT_PR --params '{"bx":128,"by":2,"merge":2,"vx":4,"pr_stages":3,"stream_chunk":128}' > gpurun_out/prof_c3.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_stream_tb_rt -s 3 -c 1 -o gpurun_out/prof_c2tb -f \
  $B --config C2 --oc ST_TB_BM_RT_PR --params '{"bx":64,"by":8,"merge":4,"vx":2,"pr_stages":3,"tb_steps":2}' > gpurun_out/prof_c2tb.log 2>&1
ls -la gpurun_out
