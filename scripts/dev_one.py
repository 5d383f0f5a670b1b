"""Dev helper: run one OC / setting on a config a few times (for ncu captures).
  python scripts/dev_one.py C2 ST_TB_RT_PR '{"tb_steps":2}' [steps] [reps]
Env STENCIL_* dev overrides apply to the codegen."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_sunlyjlq22_b200 as sm  # noqa: E402
import stencil_inputs as si  # noqa: E402

cfg, ocn = sys.argv[1], sys.argv[2]
prm = json.loads(sys.argv[3]) if len(sys.argv) > 3 else {}
steps = int(sys.argv[4]) if len(sys.argv) > 4 else 2
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 3
C = si.CONFIGS[cfg]
acc, c = si.config_stencil(os.environ.get("STENCIL_DEV_STENCIL", C["stencil"]))
dims, dtype = C["dims"], C["dtype"]
x = torch.empty(dims, dtype=torch.float64 if dtype == "f64" else torch.float32, device="cuda")
sm.fill_field(x, C["seed"])
y = torch.empty_like(x)
p = sm.Plan(dims, acc, c, dtype, ocn, prm or None)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for _ in range(reps):
    e0.record()
    p.run(x, y, steps)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    print(f"{ocn} {prm} {ms:.3f} ms {p.info['points'] * steps / ms / 1e6:.1f} GSt/s regs={p.info['regs']}", flush=True)
