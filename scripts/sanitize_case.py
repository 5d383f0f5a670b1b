"""One small run of one kernel family, checked against the oracle -- the unit
the compute-sanitizer pass (scripts/gpu_sanitize.sh) wraps:

  compute-sanitizer --tool racecheck python scripts/sanitize_case.py tbrt_split
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ipps_sunlyjlq22_b200 as sm  # noqa: E402
import stencil_inputs as si  # noqa: E402

CASES = {  # name: (stencil, dims, dtype, OC, params, steps)
    "naive": ("heat3d", (12, 20, 40), "f64", "base", None, 2),
    "tiled_tb": ("random3d:2:5", (14, 22, 40), "f64", "TB_BM", {"tb_steps": 2}, 3),
    "stream_gather": ("heat3d", (14, 20, 40), "f64", "ST_PR", None, 2),
    "stream_rt": ("random3d:2:5", (14, 20, 40), "f64", "ST_BM_RT_PR", None, 2),
    "stream_cpasync": ("heat3d", (12, 20, 37), "f64", "ST_RT_PR", None, 2),
    "stream_tb": ("heat3d", (14, 20, 40), "f64", "ST_TB_PR", None, 3),
    "tbrt_split": ("heat3d", (12, 40, 136), "f64", "ST_TB_BM_RT_PR", None, 3),
    "tbrt_xshift": ("random3d:1:0", (12, 40, 136), "f64", "ST_TB_BM_RT_PR", None, 3),
    "tbrt_cpasync": ("edge:asym3d", (12, 30, 67), "f64", "ST_TB_CM_RT_PR", None, 3),
    "tbrt_t3_fp32": ("star25", (12, 30, 72), "f32", "ST_TB_RT_PR", {"tb_steps": 3}, 4),
    "xmerge_2d": ("random2d:2:4", (40, 300), "f64", "ST_CM_RT_PR", None, 3),
    "tbrt_2d": ("random2d:1:0", (40, 300), "f64", "ST_TB_BM_RT_PR", None, 3),
    # round 2: full-width 1 x 5 intermediate tiles of k_tiled (their x-neighbour
    # reads run into the front pad / the neighbouring row), 2-D and fp32
    "tiled_tb_2d": ("random2d:2:4", (70, 300), "f64", "TB_BM", None, 3),
    "tiled_tb_fp32": ("star25", (14, 22, 72), "f32", "TB_CM", {"tb_steps": 2}, 3),
}


def run_p2p():
    """Two slabs of one grid with the fused P2P halo (edge kernels store into the
    neighbour's ghost planes, k_p2p_signal / k_p2p_wait) on two streams."""
    from paper_conf_ipps_sunlyjlq22_b200 import p2p
    acc, c = si.config_stencil("heat3d")
    gdims, steps, oc = (24, 20, 40), 3, "ST_RT_PR"
    full = torch.empty(gdims, dtype=torch.float64, device="cuda")
    sm.fill_field(full, 3)
    ref = oracle.sweep(full.cpu().numpy(), acc, c, steps)
    plans, bufs, xs, ys, wss, fl, st = [], [], [], [], [], [], []
    for k in range(2):
        z0, z1 = sm.slab_range(gdims[0], k, 2)
        p = sm.Plan((z1 - z0,) + gdims[1:], acc, c, "f64", oc)
        G = 4
        shape = (z1 - z0 + 2 * G,) + gdims[1:]
        x = torch.zeros(shape, dtype=torch.float64, device="cuda")
        a, b = max(0, z0 - G), min(gdims[0], z1 + G)
        x[a - (z0 - G):b - (z0 - G)] = full[a:b]
        xs.append(x), ys.append(torch.empty_like(x)), wss.append(torch.empty_like(x))
        fl.append(p2p.new_flags("cuda")), st.append(torch.cuda.Stream()), plans.append(p)
        bufs.append(sm.P2PBuffers(x.data_ptr(), ys[k].data_ptr(), wss[k].data_ptr(), fl[k].data_ptr(), z1 - z0))
    torch.cuda.synchronize()
    for k, p in enumerate(plans):
        p.set_p2p(k, 2, bufs[k], bufs[k - 1] if k else None, bufs[k + 1] if k < 1 else None)
        p.use_workspace(wss[k])
    for k, p in enumerate(plans):
        p.run(xs[k], ys[k], steps, stream=st[k])
    torch.cuda.synchronize()
    got = torch.cat([ys[k][4:4 + p.dims[0]] for k, p in enumerate(plans)]).cpu().numpy()
    return got, ref, "f64"


def main(name):
    if name == "p2p":
        got, ref, dtype = run_p2p()
    else:
        stn, dims, dtype, oc, prm, steps = CASES[name]
        acc, c = si.config_stencil(stn)
        u0 = si.make_field(dims, 5, dtype)
        x = torch.from_numpy(np.ascontiguousarray(u0)).cuda()
        y = torch.empty_like(x)
        p = sm.Plan(dims, acc, c, dtype, sm.oc_from_name(oc), prm)
        p.run(x, y, steps)
        torch.cuda.synchronize()
        got = y.cpu().numpy()
        ref = oracle.sweep(u0, acc, c, steps, dtype=dtype)
    err = float(np.max(np.abs(got.astype(np.float64) - ref) / np.abs(ref)))
    tol = 1e-12 if dtype == "f64" else 1e-5
    print(f"{name}: max rel err {err:.2e} ({'ok' if err <= tol else 'FAIL'})", flush=True)
    return 0 if err <= tol else 1


if __name__ == "__main__":
    sys.exit(main(sys.argv[1]))
