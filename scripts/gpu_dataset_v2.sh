# label datasets with the round-1 final kernels: 3-D at the paper's 512^3 (24 stencils), 2-D 8192^2 (40)
set -u
mkdir -p gpurun_out
timeout 2100 python scripts/label_dataset.py --out gpurun_out/ds2_3d_512.jsonl --n 24 --ndim 3 --dims 512 512 512 > gpurun_out/ds2_3d.log 2>&1
timeout 1500 python scripts/label_dataset.py --out gpurun_out/ds2_2d_8192.jsonl --n 40 --ndim 2 --dims 8192 8192 > gpurun_out/ds2_2d.log 2>&1
tail -3 gpurun_out/ds2_3d.log gpurun_out/ds2_2d.log
