"""Dev: run one OC on one small case and compare with the oracle (for sanitizer runs)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_ipps_sunlyjlq22_b200 as sm
import stencil_inputs as si
name, dims, dtype, oc = sys.argv[1], tuple(json.loads(sys.argv[2])), sys.argv[3], sys.argv[4]
prm = json.loads(sys.argv[5]) if len(sys.argv) > 5 else None
steps = 3
acc, c = si.config_stencil(name)
u0 = si.make_field(dims, 7, dtype)
ref = oracle.sweep(u0, acc, c, steps, dtype=dtype)
p = sm.Plan(dims, acc, c, dtype, sm.oc_from_name(oc), prm)
x = torch.from_numpy(u0).cuda(); y = torch.empty_like(x)
p.run(x, y, steps); torch.cuda.synchronize()
got = y.cpu().numpy()
err = float(np.max(np.abs(got - ref) / np.abs(ref)))
print(oc, p.info["params"], p.info["threads"], p.info["reg_split"], "relerr", err, flush=True)
