"""B200 analogues of the paper's Figs. 1-3 and the PCC merge into 5 classes
 from a dataset file
written by scripts/label_dataset.py.

  python scripts/oc_analysis.py gpurun_out/dataset.jsonl [--ndim 3] [--classes 5] [--json out.json]
"""
import argparse
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_conf_ipps_sunlyjlq22_b200 as sm  # noqa: E402
from paper_conf_ipps_sunlyjlq22_b200 import dataset  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("path")
ap.add_argument("--ndim", type=int, default=None)
ap.add_argument("--classes", type=int, default=5)
ap.add_argument("--json", default=None)
a = ap.parse_args()

ids, names, t = dataset.load_matrix(a.path, a.ndim)
res = sm.oc_analysis(t, a.classes)
k = len(names)
pairs = sorted(((abs(res["pcc"][i, j]), names[i], names[j]) for i in range(k) for j in range(i + 1, k)),
               key=lambda x: -x[0])
order = [int(s.split("-o")[1].split("-")[0]) if "-o" in s else 0 for s in ids]
gap = res["gap"]
out = {
    "dataset": os.path.basename(a.path), "ndim": a.ndim, "stencils": len(ids),
    "fig1_gap": {"mean": float(np.nanmean(gap)), "median": float(np.nanmedian(gap)), "max": float(np.nanmax(gap)),
                 "mean_by_order": {str(o): float(np.nanmean(gap[[i for i, x in enumerate(order) if x == o]]))
                                   for o in sorted(set(order))}},
    "fig2_wins": {n: int(w) for n, w in zip(names, res["wins"]) if w},
    "fig2_never_best": [n for n, w in zip(names, res["wins"]) if not w],
    "fig3_top_pcc": [[round(v, 4), x, y] for v, x, y in pairs[:100]],
    "groups": [[names[j] for j in range(k) if res["group"][j] == c] for c in range(max(res["group"]) + 1)],
    "representatives": [names[r] for r in res["representative"]],
    "class_histogram": np.bincount([c for c in res["labels"] if c >= 0], minlength=a.classes).tolist(),
    "infeasible_per_oc": {n: int(np.sum(~np.isfinite(t[:, j]))) for j, n in enumerate(names)
                          if np.any(~np.isfinite(t[:, j]))},
}
txt = json.dumps(out, indent=1)
if a.json:
    with open(a.json, "w") as f:
        f.write(txt + "\n")
print(json.dumps({k2: out[k2] for k2 in ("stencils", "fig1_gap", "fig2_wins", "representatives", "class_histogram")}))
