#!/bin/bash
# ncu --set full of the TB kernels at 2 fused steps (dev_prof_one STEPS = 2), and 2-D TB tile heights
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for spec in "c5_r1 C5 random3d:1:0 ST_TB_BM_RT_PR k_stream_tb_rt {}" "c2 C2 heat3d ST_TB_BM_RT_PR k_stream_tb_rt {}" \
            "n2_r2 N2 random2d:2:4 TB_BM k_tiled {}" "n2_r2_by8 N2 random2d:2:4 TB_BM k_tiled {\"by\":8}" \
            "n2_r1 N2 random2d:1:0 TB_BM k_tiled {}"; do
  set -- $spec
  ncu --set full --import-source on --clock-control none -k regex:$5 -s 2 -c 1 -o gpurun_out/r02d_$1_full \
      python scripts/dev_prof_one.py $2 $3 $4 "$6" 2 > gpurun_out/r02d_$1_full.log 2>&1
  echo "$1 rc=$?"
done
for st in random2d:1:0 random2d:2:4; do
  timeout 600 python scripts/dev_tune.py --cfg N2 --stencil $st --ocs TB_BM,TB_CM,TB --steps 10 --top 20 \
    --grid '{"bx":[64,128],"by":[4,8,16],"vx":[2],"merge":[1,4],"tb_steps":[2]}' > gpurun_out/tune_n2_${st//:/_}_by.log 2>&1
done
