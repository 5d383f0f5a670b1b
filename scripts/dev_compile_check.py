"""Dev tool (CPU): NVRTC-compile plans and print register / spill use of the
cached cubins (cuobjdump -res-usage). Usage:
  python scripts/dev_compile_check.py heat3d:f64:ST_TB_RT[:json-params] ...
"""
import glob
import json
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_sunlyjlq22_b200 as sm  # noqa: E402
import stencil_inputs as si  # noqa: E402

CACHE = os.path.expanduser("~/.cache/stencilmart")


def newest_cubin():
    fs = glob.glob(os.path.join(os.environ.get("STENCIL_CACHE_DIR", CACHE), "*.cubin"))
    return max(fs, key=os.path.getmtime) if fs else None


for spec in sys.argv[1:]:
    parts = spec.split(":", 3)
    name, dtype, oc = parts[0], parts[1], parts[2]
    rest = parts[3] if len(parts) > 3 else ""
    if name == "random3d" or name == "random2d":   # random3d:order:seed packed as name-order-seed
        pass
    prm = json.loads(rest) if rest else None
    sname = name.replace("-", ":")
    acc, c = si.config_stencil(sname)
    dims = (64, 64, 64) if acc.ndim == 3 else (256, 256)
    import tempfile
    CACHE = tempfile.mkdtemp(prefix="smcc")
    os.environ["STENCIL_CACHE_DIR"] = CACHE
    try:
        p = sm.Plan(dims, acc, c, dtype, sm.oc_from_name(oc), prm)
    except sm.StencilError as e:
        print(spec, "->", "ERR", e)
        continue
    cub = newest_cubin()
    usage = ""
    if cub:
        out = subprocess.run(["cuobjdump", "-res-usage", cub], capture_output=True, text=True).stdout
        usage = " ".join(line.strip() for line in out.splitlines() if "REG" in line)
    print(spec, "->", p.info["params"], "|", usage[:300])
