"""Dev helper: time each OC on a config with CUDA events (not the bench)."""
import argparse, json, sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_sunlyjlq22_b200 as sm
import stencil_inputs as si

ap = argparse.ArgumentParser()
ap.add_argument("--cfg", default="C2")
ap.add_argument("--ocs", default="all")
ap.add_argument("--steps", type=int, default=10)
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--params", default="{}")
ap.add_argument("--stencil", default="")
a = ap.parse_args()
C = si.CONFIGS[a.cfg]
acc, c = si.config_stencil(a.stencil or (C["stencil"] if C["stencil"] != "random3d" else "random3d:2:1"))
dims, dtype = C["dims"], C["dtype"]
tdt = torch.float64 if dtype == "f64" else torch.float32
x = torch.empty(dims, dtype=tdt, device="cuda"); sm.fill_field(x, C["seed"])
y = torch.empty_like(x)
elem = 8 if dtype == "f64" else 4
ocs = sm.oc_list() if a.ocs == "all" else [sm.oc_from_name(n) for n in a.ocs.split(",")]
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for oc in ocs:
    t = time.time()
    try:
        p = sm.Plan(dims, acc, c, dtype, oc, json.loads(a.params))
    except sm.StencilError as e:
        print(f"{sm.oc_name(oc):16s} infeasible: {str(e)[:100]}"); continue
    ct = time.time() - t
    p.run(x, y, a.steps); torch.cuda.synchronize()
    best = 1e9
    for _ in range(a.reps):
        e0.record(); p.run(x, y, a.steps); e1.record(); torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    i = p.info
    gs = i["points"] * a.steps / (best * 1e-3) / 1e9
    bw = gs * 2 * elem
    print(f"{sm.oc_name(oc):16s} {best:8.3f} ms  {gs:7.1f} GSt/s  {bw:7.1f} GB/s  fam={i['family']} thr={i['threads']} smem={i['smem_bytes']} regs={i['regs']} tma={i['uses_tma']} compile={ct:.1f}s", flush=True)
