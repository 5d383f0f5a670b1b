#!/bin/bash
# ncu --set full (with source) of C2's dominant kernel, k_stream_tb_rt at the
# default setting of ST_TB_BM_RT_PR (the OC the C2 label pass picks). Usage under
# gpurun: bash scripts/gpu_prof_c2.sh <tag> [extra env assignments...]
tag=${1:-c2}
shift
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
env "$@" ncu --set full --import-source on --clock-control none -k regex:k_stream_tb_rt -s 4 -c 1 \
    -o gpurun_out/${tag} python bench.py --config C2 --oc ST_TB_BM_RT_PR --steps 1 --warmup 3 --no-cpu --no-e2e \
    > gpurun_out/${tag}_prof.log 2>&1
echo "ncu rc=$?"
