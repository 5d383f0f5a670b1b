#!/bin/bash
# label datasets with the round-2 final kernels: 60 3-D Algorithm-1 stencils at 512^3, 80 2-D at 8192^2 (resumable)
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 2400 python scripts/label_dataset.py --out gpurun_out/ds3_3d_512.jsonl --n 60 --ndim 3 --dims 512 512 512 > gpurun_out/ds3_3d.log 2>&1
timeout 1500 python scripts/label_dataset.py --out gpurun_out/ds3_2d_8192.jsonl --n 80 --ndim 2 --dims 8192 8192 > gpurun_out/ds3_2d.log 2>&1
tail -3 gpurun_out/ds3_3d.log gpurun_out/ds3_2d.log
