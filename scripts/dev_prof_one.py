"""Dev: run one OC of one stencil on a config's grid a few times (ncu target).

  python scripts/dev_prof_one.py CFG STENCIL OC [PARAMS_JSON] [STEPS]
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_sunlyjlq22_b200 as sm
import stencil_inputs as si
cfg, stencil, oc = sys.argv[1], sys.argv[2], sys.argv[3]
prm = json.loads(sys.argv[4]) if len(sys.argv) > 4 and sys.argv[4] else None
steps = int(sys.argv[5]) if len(sys.argv) > 5 else 1
C = si.CONFIGS[cfg]
acc, c = si.config_stencil(stencil)
tdt = torch.float64 if C["dtype"] == "f64" else torch.float32
x = torch.empty(C["dims"], dtype=tdt, device="cuda"); sm.fill_field(x, C["seed"])
y = torch.empty_like(x)
p = sm.Plan(C["dims"], acc, c, C["dtype"], sm.oc_from_name(oc), prm)
for _ in range(3):
    p.run(x, y, steps)
torch.cuda.synchronize()
print(p.info["kernel_name"], p.info["params"], p.info["regs"])
