"""Label random Algorithm-1 stencils on this GPU (the paper's dataset).

  python scripts/label_dataset.py --out gpurun_out/dataset.jsonl --n 8 --ndim 3 --dims 256 256 256

Resumable: stencils already labelled in --out are skipped.
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import stencil_inputs as si  # noqa: E402
from paper_conf_ipps_sunlyjlq22_b200 import dataset  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--out", required=True)
ap.add_argument("--n", type=int, default=8, help="stencils (orders cycle 1..4)")
ap.add_argument("--ndim", type=int, default=3)
ap.add_argument("--dims", type=int, nargs="+", default=[256, 256, 256])
ap.add_argument("--dtype", default="f64")
ap.add_argument("--steps", type=int, default=4)
ap.add_argument("--settings", type=int, default=3)
ap.add_argument("--seed", type=int, default=0)
a = ap.parse_args()
done = dataset.resume(a.out)      # cut a torn tail of an interrupted run
for i in range(a.n):
    order = 1 + i % 4
    sid = f"{a.ndim}d-o{order}-s{a.seed + i}"
    if sid in done:
        continue
    acc, _ = si.random_stencil(a.ndim, order, a.seed + i)
    c = si.random_coeffs(acc, a.seed + i)
    t0 = time.time()
    rows = dataset.label_stencil(sid, acc, c, a.dims, a.dtype, a.steps, a.settings, seed=a.seed)
    dataset.append_rows(a.out, rows)
    lab = rows[-1]
    print(f"{sid}: nnz={lab['features']['nnz']} best={lab['best_oc_name']} ({time.time() - t0:.1f} s)", flush=True)
