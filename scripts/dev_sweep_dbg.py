import sys, os, math
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_sunlyjlq22_b200 as sm
import stencil_inputs as si
acc, c = si.config_stencil("random3d:1:4")
dims = (40, 40, 64)
x = torch.empty(dims, dtype=torch.float64, device="cuda"); sm.fill_field(x, 3)
y = torch.empty_like(x)
only = sys.argv[1] if len(sys.argv) > 1 else None
for oc in sm.oc_list():
    for k in range(2):
        prm = sm.sample_params(oc, 3, "f64", 7, k)
        if only and sm.oc_name(oc) != only: continue
        try:
            p = sm.Plan(dims, acc, c, "f64", oc, prm)
        except sm.StencilError as e:
            print(sm.oc_name(oc), k, "skip", e.name); continue
        print(sm.oc_name(oc), k, prm, p.info["kernel_name"][:80], flush=True)
        p.run(x, y, 2); torch.cuda.synchronize()
print("ok")
