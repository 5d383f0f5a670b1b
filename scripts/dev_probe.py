import sys, os, json, subprocess
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if len(sys.argv) > 2:
    import torch, numpy as np
    import paper_conf_ipps_sunlyjlq22_b200 as sm, stencil_inputs as si
    name, oc, prm = sys.argv[1], sys.argv[2], json.loads(sys.argv[3])
    acc, c = si.config_stencil(name)
    dims = tuple(json.loads(sys.argv[4])) if len(sys.argv) > 4 else (40, 40, 64)
    x = torch.empty(dims, dtype=torch.float64, device="cuda"); sm.fill_field(x, 3)
    y = torch.empty_like(x)
    p = sm.Plan(dims, acc, c, "f64", sm.oc_from_name(oc), prm)
    p.run(x, y, 2); torch.cuda.synchronize(); print("OK", p.info["kernel_name"][:90]); sys.exit(0)
cases = json.loads(sys.argv[1])
for cse in cases:
    r = subprocess.run([sys.executable, __file__] + [str(a) if not isinstance(a, (dict, list)) else json.dumps(a) for a in cse], capture_output=True, text=True)
    last = (r.stdout.strip().splitlines() or [""])[-1] + (r.stderr.strip().splitlines() or [""])[-1]
    print(cse, "->", last[:200], flush=True)
