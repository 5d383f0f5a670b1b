"""Dev helper: grid-search parameter settings of some OCs on a config (CUDA events)."""
import argparse
import itertools
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_sunlyjlq22_b200 as sm  # noqa: E402
import stencil_inputs as si  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--cfg", default="C2")
ap.add_argument("--ocs", default="ST_PR")
ap.add_argument("--grid", default='{"bx":[64,128],"by":[4,8],"vx":[2],"merge":[1],"stream_chunk":[64,128,256],"pr_stages":[2,3,4]}')
ap.add_argument("--steps", type=int, default=4)
ap.add_argument("--top", type=int, default=12)
ap.add_argument("--stencil", default="")
a = ap.parse_args()
C = si.CONFIGS[a.cfg]
acc, c = si.config_stencil(a.stencil or C["stencil"])
dims, dtype = C["dims"], C["dtype"]
tdt = torch.float64 if dtype == "f64" else torch.float32
x = torch.empty(dims, dtype=tdt, device="cuda")
sm.fill_field(x, C["seed"])
y = torch.empty_like(x)
elem = 8 if dtype == "f64" else 4
grid = json.loads(a.grid)
keys = list(grid)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
res = []
for ocn in a.ocs.split(","):
    for vals in itertools.product(*[grid[k] for k in keys]):
        prm = dict(zip(keys, vals))
        for k in list(prm):           # "env:MINB": 3 -> STENCIL_MINB=3 for this plan's codegen
            if k.startswith("env:"):
                os.environ["STENCIL_" + k[4:]] = str(prm.pop(k))
        shown = dict(zip(keys, vals))
        try:
            p = sm.Plan(dims, acc, c, dtype, ocn, prm)
            p.run(x, y, a.steps)
            torch.cuda.synchronize()
            best = 1e9
            for _ in range(3):
                e0.record()
                p.run(x, y, a.steps)
                e1.record()
                torch.cuda.synchronize()
                best = min(best, e0.elapsed_time(e1))
        except sm.StencilError as e:
            continue
        pts = p.info["points"]
        gs = pts * a.steps / (best * 1e-3) / 1e9
        res.append((gs, ocn, shown, p.info["regs"], p.info["smem_bytes"]))
        print(f"{ocn:14s} {gs:7.1f} GSt/s {gs * 2 * elem:7.0f} GB/s regs={p.info['regs']} smem={p.info['smem_bytes']} {shown}",
              flush=True)
        del p
res.sort(key=lambda r: -r[0])
print("=== top")
for r in res[: a.top]:
    print(f"{r[1]:14s} {r[0]:7.1f} GSt/s {r[0] * 2 * elem:7.0f} GB/s regs={r[3]} smem={r[4]} {r[2]}")
