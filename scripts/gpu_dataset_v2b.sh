# extend the round-1 label datasets (resumable JSONL): 3-D 512^3 to 60 stencils, 2-D 8192^2 to 80
set -u
mkdir -p gpurun_out
cp ds_in/ds2_3d_512.jsonl gpurun_out/ds2_3d_512.jsonl; cp ds_in/ds2_2d_8192.jsonl gpurun_out/ds2_2d_8192.jsonl
timeout 1800 python scripts/label_dataset.py --out gpurun_out/ds2_3d_512.jsonl --n 60 --ndim 3 --dims 512 512 512 > gpurun_out/ds2b_3d.log 2>&1
timeout 1200 python scripts/label_dataset.py --out gpurun_out/ds2_2d_8192.jsonl --n 80 --ndim 2 --dims 8192 8192 > gpurun_out/ds2b_2d.log 2>&1
wc -l gpurun_out/ds2_3d_512.jsonl gpurun_out/ds2_2d_8192.jsonl
