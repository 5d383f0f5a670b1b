#!/bin/bash
# round-2 batch 2: ncu source-level profile of C2's k_stream_tb_rt, N2 2-D TB tile
# shapes, FP64 FMA probe variants
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/fmaprobe scripts/dev_fma_probe.cu && /tmp/fmaprobe > gpurun_out/fmaprobe.log 2>&1
T="python scripts/dev_time.py"
for st in random2d:1:0 random2d:2:4; do
  for prm in '{}' '{"bx":128}' '{"by":8}' '{"bx":128,"by":8}' '{"merge":8}' '{"bx":128,"merge":8}' '{"tb_steps":4}'; do
    echo "-- $st $prm"; $T --cfg N2 --stencil $st --ocs TB_BM,TB_CM --reps 3 --params "$prm"
  done
done > gpurun_out/ab_n2tb.log 2>&1
bash scripts/gpu_prof_c2.sh r02_c2_tbrt
