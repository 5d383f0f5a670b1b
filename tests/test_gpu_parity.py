"""GPU parity: every OC's CUDA path (through the C ABI) against the oracle.

Bars (BASELINE.json north_star): fp64 max relative error <= 1e-12, fp32 <= 1e-5
after the sweep; dyadic-exact inputs bitwise equal to the oracle; all OCs
bitwise equal to each other (canonical FMA order); integer outputs
(OC ids, label) bit-exact.
"""
import concurrent.futures as cf
import math

import os

import numpy as np
import pytest

import oracle
import paper_conf_ipps_sunlyjlq22_b200 as sm
import stencil_inputs as si

pytestmark = pytest.mark.gpu

TOL = {"f64": 1e-12, "f32": 1e-5}


def _torch():
    import torch
    return torch


def _to_dev(a, dtype):
    torch = _torch()
    t = torch.from_numpy(np.ascontiguousarray(a.astype(np.float64 if dtype == "f64" else np.float32)))
    return t.cuda()


def _plans(acc, c, dims, dtype, ocs, params=None):
    """Create (NVRTC-compile) plans in parallel threads; infeasible -> None."""
    def mk(oc):
        try:
            return sm.Plan(dims, acc, c, dtype, oc, params)
        except sm.StencilError as e:
            if e.code == -3:
                return None
            raise
    with cf.ThreadPoolExecutor(os.cpu_count() or 8) as ex:
        return dict(zip(ocs, ex.map(mk, ocs)))


def _run(plan, u0, dtype, steps):
    torch = _torch()
    x = _to_dev(u0, dtype)
    y = torch.empty_like(x)
    plan.run(x, y, steps)
    torch.cuda.synchronize()
    return y.cpu().numpy()


def _relerr(got, ref):
    return float(np.max(np.abs(got.astype(np.float64) - ref) / np.maximum(np.abs(ref), 1e-300)))


CASES = [
    # (stencil, dims (ragged vs tiles), dtype, steps): 10 steps, the north-star bar
    ("heat3d", (37, 45, 70), "f64", 10),
    ("heat3d", (33, 29, 67), "f64", 10),          # rows not 16-B multiples: cp.async staging
    ("heat3d", (36, 41, 68), "f32", 10),
    ("star25", (30, 27, 72), "f32", 10),
    ("box125", (22, 26, 40), "f64", 10),
    ("random3d:1:2", (29, 31, 38), "f64", 10),
    ("random3d:2:5", (27, 33, 44), "f64", 10),
    ("random3d:3:1", (24, 26, 36), "f32", 10),
    ("random3d:4:3", (25, 23, 40), "f64", 10),
    # NEXT-2: random 2-D stencils (Algorithm 1, d = 2) under all 30 OCs; the
    # streaming OCs stream along y (C-13)
    ("random2d:1:0", (70, 90), "f64", 10),
    ("random2d:2:4", (45, 130), "f64", 10),
    ("random2d:3:8", (61, 77), "f32", 10),
    ("random2d:4:12", (50, 68), "f64", 10),
]


@pytest.mark.parametrize("name,dims,dtype,steps", CASES)
def test_every_oc_matches_oracle(gpu, name, dims, dtype, steps):
    acc, c = si.config_stencil(name)
    u0 = si.make_field(dims, 11, dtype)
    ref = oracle.sweep(u0, acc, c, steps, dtype=dtype)
    ocs = sm.oc_list()
    plans = _plans(acc, c, dims, dtype, ocs)
    base = None
    ran = []
    for oc in ocs:
        p = plans[oc]
        if p is None:
            continue
        got = _run(p, u0, dtype, steps)
        err = _relerr(got, ref)
        assert err <= TOL[dtype], (sm.oc_name(oc), err, p.info["kernel_name"])
        if base is None:
            base = got
        else:   # canonical FMA order: every OC bitwise identical (P9)
            assert np.array_equal(got, base), (sm.oc_name(oc), float(np.max(np.abs(got - base))))
        ran.append(sm.oc_name(oc))
    assert "base" in ran and "ST" in ran and "ST_RT" in ran and len(ran) >= 14, ran


@pytest.mark.parametrize("name,dtype,steps", [("heat3d", "f64", 10), ("box125", "f64", 6),
                                              ("star25", "f32", 2), ("heat2d", "f64", 10)])
def test_dyadic_bitwise(gpu, name, dtype, steps):
    acc, c = si.config_stencil(name)
    dims = (26, 30, 44) if acc.ndim == 3 else (60, 72)
    u0 = si.make_field(dims, 5, dtype, kind="int1023")
    ref = oracle.sweep(u0, acc, c, steps, dtype=dtype)
    ocs = [0, sm.OC_ST, sm.OC_ST | sm.OC_RT, sm.OC_TB, sm.OC_ST | sm.OC_BM | sm.OC_PR]
    for oc, p in _plans(acc, c, dims, dtype, ocs).items():
        if p is None:
            continue
        got = _run(p, u0, dtype, steps).astype(np.float64)
        assert np.array_equal(got, ref), sm.oc_name(oc)


def test_2d_heat_c1(gpu):
    """C1: 2-D 5-point star, 256^2 fp64, 10 steps, naive OC."""
    acc, c = si.heat2d()
    u0 = si.make_field((256, 256), 0xC0FFEE + 1, "f64")
    ref = oracle.sweep(u0, acc, c, 10)
    for oc in (0, sm.OC_ST, sm.OC_BM, sm.OC_TB):
        got = _run(sm.Plan((256, 256), acc, c, "f64", oc), u0, "f64", 10)
        assert _relerr(got, ref) <= 1e-12, sm.oc_name(oc)


def test_parameter_settings(gpu):
    """Sampled settings of several OCs (other tile shapes, merge factors, T)."""
    acc, c = si.config_stencil("random3d:2:7")
    dims, dtype, steps = (30, 34, 52), "f64", 3
    u0 = si.make_field(dims, 3, dtype)
    ref = oracle.sweep(u0, acc, c, steps)
    for oc in (0, sm.OC_BM, sm.OC_TB | sm.OC_CM, sm.OC_ST | sm.OC_CM | sm.OC_RT, sm.OC_ST | sm.OC_PR):
        for k in range(1, 4):
            prm = sm.sample_params(oc, 3, dtype, 99, k)
            try:
                p = sm.Plan(dims, acc, c, dtype, oc, prm)
            except sm.StencilError as e:
                assert e.code == -3
                continue
            got = _run(p, u0, dtype, steps)
            assert _relerr(got, ref) <= 1e-12, (sm.oc_name(oc), prm)


def test_fill_field_matches_generator(gpu):
    torch = _torch()
    for dtype, kind in [("f64", 0), ("f32", 0), ("f64", 1)]:
        t = torch.empty((7, 9, 11), dtype=torch.float64 if dtype == "f64" else torch.float32, device="cuda")
        sm.fill_field(t, 123, kind, origin=(2, 3, 4), global_dims=(20, 30, 40))
        torch.cuda.synchronize()
        ref = si.make_field((7, 9, 11), 123, dtype, si.KINDS[kind], origin=(2, 3, 4), global_dims=(20, 30, 40))
        assert np.array_equal(t.cpu().numpy(), ref)


def test_steps_zero_and_errors(gpu):
    torch = _torch()
    acc, c = si.heat3d()
    p = sm.Plan((12, 12, 16), acc, c, "f64", sm.OC_ST)
    x = torch.rand((12, 12, 16), dtype=torch.float64, device="cuda")
    y = torch.empty_like(x)
    p.run(x, y, 0)
    torch.cuda.synchronize()
    assert torch.equal(x, y)
    with pytest.raises(sm.StencilError):
        p.run(x, x, 1)


def test_run_host_end_to_end(gpu):
    acc, c = si.star25()
    dims = (24, 20, 36)
    u0 = si.make_field(dims, 8, "f32")
    p = sm.Plan(dims, acc, c, "f32", sm.OC_ST | sm.OC_RT)
    out = np.empty(dims, np.float32)
    p.run_host(np.ascontiguousarray(u0), out, 3)
    ref = oracle.sweep(u0, acc, c, 3, dtype="f32")
    assert _relerr(out, ref) <= 1e-5


def test_run_host_small_grid_not_pipelined(gpu):
    """C1-sized grids (256^2 fp64, 0.5 MB) stay on the unpipelined host path:
    per-chunk copy/launch latency would exceed the overlap (api.cpp
    run_host_pipelined size threshold)."""
    acc, c = si.heat2d()
    dims = (256, 256)
    u0 = np.ascontiguousarray(si.make_field(dims, 3, "f64"))
    p = sm.Plan(dims, acc, c, "f64", sm.OC_ST | sm.OC_RT)
    out = np.empty_like(u0)
    p.run_host(u0, out, 10)
    assert p.info["host_chunks"] == 0
    ref = oracle.sweep(u0, acc, c, 10, dtype="f64")
    assert _relerr(out, ref) <= 1e-12


@pytest.mark.parametrize("name,dims,dtype,oc,prm,steps", [
    ("heat3d", (160, 40, 72), "f64", "ST_TB_BM_RT_PR", None, 5),      # TB with a remainder launch
    ("heat3d", (130, 33, 64), "f64", "base", None, 4),
    ("random3d:2:5", (150, 36, 48), "f64", "ST_BM_RT_PR", None, 3),
    ("random3d:1:0", (140, 40, 80), "f64", "ST_TB_CM_RT", {"merge": 2}, 6),
    ("star25", (200, 30, 72), "f32", "ST_RT_PR", None, 2),
    ("box125", (128, 26, 40), "f64", "TB_BM", {"tb_steps": 2}, 3),
    ("random2d:3:8", (700, 90), "f64", "ST_BM_RT_PR", None, 4),
    # 2-D tiled / naive views [1][ny][nx] chunk along y
    ("random2d:1:0", (600, 130), "f64", "TB_BM", None, 5),
    ("random2d:2:4", (300, 100), "f64", "base", None, 3)])
def test_run_host_pipelined(gpu, name, dims, dtype, oc, prm, steps):
    """stencil_run_host pipelines H2D / sweep / D2H over z-chunks with a
    time-skewed wavefront (api.cpp run_host_pipelined): bitwise equal to the
    device-buffer run and to the unpipelined host path, and within tolerance
    of the oracle."""
    torch = _torch()
    acc, c = si.config_stencil(name)
    u0 = np.ascontiguousarray(si.make_field(dims, 17, dtype))
    p = sm.Plan(dims, acc, c, dtype, sm.oc_from_name(oc), prm)
    out = np.empty_like(u0)
    os.environ["STENCIL_PIPELINE_MIN_BYTES"] = "0"     # these grids are below the size threshold
    try:
        p.run_host(u0, out, steps)
    finally:
        del os.environ["STENCIL_PIPELINE_MIN_BYTES"]
    assert p.info["host_chunks"] >= 2          # the pipelined path ran
    dev = _run(p, u0, dtype, steps)
    assert np.array_equal(out, dev)
    os.environ["STENCIL_NO_PIPELINE"] = "1"
    try:
        out2 = np.empty_like(u0)
        sm.Plan(dims, acc, c, dtype, sm.oc_from_name(oc), prm).run_host(u0, out2, steps)
    finally:
        del os.environ["STENCIL_NO_PIPELINE"]
    assert np.array_equal(out, out2)
    ref = oracle.sweep(u0, acc, c, steps, dtype=dtype)
    assert _relerr(out, ref) <= TOL[dtype]


def test_oc_sweep_label(gpu):
    torch = _torch()
    acc, c = si.config_stencil("random3d:1:4")
    dims = (40, 40, 64)
    x = torch.empty(dims, dtype=torch.float64, device="cuda")
    sm.fill_field(x, 3)
    y = torch.empty_like(x)
    p = sm.Plan(dims, acc, c, "f64", 0)
    res = p.oc_sweep(x, y, steps=2, settings_per_oc=2, reps=3, seed=7)
    assert res["oc_ids"] == oracle.valid_ocs()
    assert res["best_oc"] == oracle.best_oc(res["times_ms"], res["oc_ids"])
    assert sum(math.isfinite(t) for t in res["times_ms"]) >= 14
    # the output of the sweep is a correct sweep
    ref = oracle.sweep(x.cpu().numpy(), acc, c, 2)
    assert _relerr(y.cpu().numpy(), ref) <= 1e-12


@pytest.mark.parametrize("cfg,ocs,stencil", [
    ("C2", ["ST_RT_PR", "ST_PR", "base", "ST_TB_BM_RT_PR"], None),
    ("C3", ["ST_RT_PR", "ST_BM_RT_PR", "ST_CM_RT_PR"], None),
    ("C4", ["ST_RT_PR", "TB", "ST_CM_RT_PR"], None), ("C5", ["ST_BM_RT_PR"], "random3d:4:12"),
    ("C5", ["ST_TB_BM_RT_PR"], "random3d:1:0"), ("C5", ["ST_BM_RT_PR", "ST_CM_RT_PR"], "random3d:2:4"),
    ("N2", ["TB_BM", "ST_BM_RT_PR"], "random2d:3:8"), ("N2", ["TB_BM"], "random2d:1:0"),
    ("N2", ["ST_RT_PR", "TB_BM"], "random2d:4:12")])
def test_full_size_sampled(gpu, cfg, ocs, stencil):
    """BASELINE sizes, the bench's launch configuration (default settings of
    the OCs the bench labels), sampled points vs the oracle on their
    dependency cones."""
    torch = _torch()
    C = si.CONFIGS[cfg]
    acc, c = si.config_stencil(stencil or C["stencil"])
    dims, dtype, steps = C["dims"], C["dtype"], C["steps"]
    tdt = torch.float64 if dtype == "f64" else torch.float32
    x = torch.empty(dims, dtype=tdt, device="cuda")
    sm.fill_field(x, C["seed"])
    y = torch.empty_like(x)
    rng = np.random.default_rng(0)
    pts = np.stack([rng.integers(0, n, size=24) for n in dims], axis=1)
    nd = len(dims)
    edge = [[0] * nd, [4] * nd, [d - 5 for d in dims[:-1]] + [dims[-1] - 6],       # frame, near-frame
            [dims[0] // 2] + [4] * (nd - 2) + [dims[-1] - 5], [d - 1 for d in dims]]
    pts = np.concatenate([pts, np.array(edge, dtype=pts.dtype)])
    ref = oracle.sweep_points(pts, dims, C["seed"], "uniform12", acc, c, steps, dtype)
    for name in ocs:
        p = sm.Plan(dims, acc, c, dtype, sm.oc_from_name(name))
        p.run(x, y, steps)
        torch.cuda.synchronize()
        got = y[tuple(torch.from_numpy(pts.T).cuda())].cpu().numpy()
        assert _relerr(got, ref) <= TOL[dtype], name
        del p
    del x, y
    torch.cuda.empty_cache()


@pytest.mark.parametrize("name,dims,dtype", [("heat3d", (41, 37, 70), "f64"), ("random3d:2:5", (29, 31, 44), "f64"),
                                             ("star25", (36, 30, 72), "f32"), ("box125", (26, 28, 40), "f64")])
def test_tb_rt_pipeline_settings(gpu, name, dims, dtype):
    """Warp-specialised ST_TB_RT pipeline (k_stream_tb_rt): fused depths 2..4,
    several z-chunks per column (stream_chunk), merge modes, prefetch depths
    1..4, and a step count that leaves a TB remainder launch."""
    acc, c = si.config_stencil(name)
    steps = 5
    u0 = si.make_field(dims, 21, dtype)
    ref = oracle.sweep(u0, acc, c, steps, dtype=dtype)
    base = _run(sm.Plan(dims, acc, c, dtype, 0), u0, dtype, steps)
    settings = [("ST_TB_RT", {"tb_steps": 2, "stream_chunk": 8}),
                ("ST_TB_RT_PR", {"tb_steps": 3, "pr_stages": 4, "stream_chunk": 16}),
                ("ST_TB_BM_RT_PR", {"tb_steps": 4, "merge": 2, "pr_stages": 2}),
                ("ST_TB_CM_RT", {"tb_steps": 2, "merge": 4, "by": 4}),
                ("ST_TB_BM_RT", {"tb_steps": 3, "merge": 8, "by": 2, "bx": 32})]
    ran = 0
    for oc, prm in settings:
        try:
            p = sm.Plan(dims, acc, c, dtype, sm.oc_from_name(oc), prm)
        except sm.StencilError as e:
            assert e.code == -3, (oc, prm, str(e))
            continue
        got = _run(p, u0, dtype, steps)
        assert _relerr(got, ref) <= TOL[dtype], (oc, prm)
        assert np.array_equal(got, base), (oc, prm)
        ran += 1
    assert ran >= 3


def test_tb_rt_xshift_remainder(gpu):
    """T = 4 aligned-window plan run for 7 steps: the remainder launch of depth 3
    would start its TMA box 3 columns (24 bytes) left of the tile -- misaligned --
    so it takes the rounded geometry; the result must still match."""
    acc, c = si.config_stencil("random3d:1:0")
    dims = (30, 50, 96)
    u0 = si.make_field(dims, 41, "f64")
    ref = oracle.sweep(u0, acc, c, 7, dtype="f64")
    base = _run(sm.Plan(dims, acc, c, "f64", 0), u0, "f64", 7)
    p = sm.Plan(dims, acc, c, "f64", sm.oc_from_name("ST_TB_BM_RT_PR"), {"tb_steps": 4, "merge": 2})
    assert p.info["xshift"]
    got = _run(p, u0, "f64", 7)
    assert _relerr(got, ref) <= TOL["f64"]
    assert np.array_equal(got, base)


@pytest.mark.parametrize("name,dims,dtype,oc,prm", [
    ("heat3d", (20, 100, 200), "f64", "ST_TB_BM_RT_PR", None),
    ("heat3d", (21, 90, 170), "f64", "ST_TB_CM_RT", {"merge": 4, "by": 4}),
    ("star25", (24, 80, 300), "f32", "ST_TB_RT_PR", None),
    ("random3d:2:5", (22, 70, 140), "f64", "ST_TB_BM_RT_PR", {"tb_steps": 3, "merge": 2}),
    # order-1 Algorithm-1 stencils take the aligned-window ring geometry (xshift)
    ("random3d:1:0", (20, 100, 200), "f64", "ST_TB_BM_RT_PR", None),
    # T = 4 with xshift: 4 steps in one launch (the remainder-depth guard is in
    # test_tb_rt_xshift_remainder)
    ("random3d:1:2", (24, 60, 140), "f64", "ST_TB_BM_RT_PR", {"tb_steps": 4, "merge": 2}),
    ("random3d:1:1", (23, 75, 150), "f64", "ST_TB_CM_RT_PR", {"merge": 2, "by": 8})])
def test_tb_rt_interior_and_edge_tiles(gpu, name, dims, dtype, oc, prm):
    """k_stream_tb_rt on grids large enough that some tiles lie wholly inside
    the compute box next to edge tiles (frame values of the intermediate step
    come from the input ring); element-wise vs the oracle, bitwise vs OC base."""
    acc, c = si.config_stencil(name)
    steps = 4
    u0 = si.make_field(dims, 31, dtype)
    ref = oracle.sweep(u0, acc, c, steps, dtype=dtype)
    base = _run(sm.Plan(dims, acc, c, dtype, 0), u0, dtype, steps)
    got = _run(sm.Plan(dims, acc, c, dtype, sm.oc_from_name(oc), prm), u0, dtype, steps)
    assert _relerr(got, ref) <= TOL[dtype]
    assert np.array_equal(got, base)


def test_sweep_rows(gpu):
    """NEXT-1: the label generator's rows (stencil_sweep_rows; "each
    parameter setting and its corresponding execution time are also stored"):
    30 x K rows in sweep order (OC ids ascending, settings 0..K-1); each row's
    setting is the resolved stencil_sample_params(seed, oc, k) (k = 0: the
    defaults), or the raw sample when the setting is infeasible; per OC the
    label time is the minimum over its rows (bit-exact) and best_params the
    first argmin row."""
    torch = _torch()
    acc, c = si.config_stencil("random3d:2:6")
    dims, dtype, K, seed = (36, 40, 56), "f64", 3, 11
    x = torch.empty(dims, dtype=torch.float64, device="cuda")
    sm.fill_field(x, 4)
    y = torch.empty_like(x)
    res = sm.Plan(dims, acc, c, dtype, 0).oc_sweep(x, y, steps=2, settings_per_oc=K, reps=3, seed=seed)
    rows = res["rows"]
    ids = oracle.valid_ocs()
    assert res["oc_ids"] == ids and len(rows) == len(ids) * K
    for i, oc in enumerate(ids):
        rr = rows[i * K:(i + 1) * K]
        assert [r["oc"] for r in rr] == [oc] * K and [r["setting"] for r in rr] == list(range(K))
        for k, r in enumerate(rr):
            raw = sm.sample_params(oc, 3, dtype, seed, k)
            if math.isfinite(r["time_ms"]):
                want = sm.Plan(dims, acc, c, dtype, oc, None if k == 0 else raw).info["params"]
            else:
                want = raw
            assert r["params"] == want, (sm.oc_name(oc), k)
        ts = [r["time_ms"] for r in rr]
        fin = [t for t in ts if math.isfinite(t)]
        if not fin:
            assert not math.isfinite(res["times_ms"][i])
            continue
        assert res["times_ms"][i] == min(fin), sm.oc_name(oc)
        assert res["best_params"][i] == rr[ts.index(min(fin))]["params"], sm.oc_name(oc)
    assert res["best_oc"] == oracle.best_oc(res["times_ms"], res["oc_ids"])


@pytest.mark.parametrize("cfg,oc", [("C2", "ST_TB_BM_RT_PR"), ("C2", "ST_RT_PR"), ("C4", "ST_CM_RT_PR"),
                                    ("C4", "ST_BM_RT_PR")])
def test_full_grid_elementwise(gpu, cfg, oc):
    """BASELINE sizes, whole grid, element by element against the oracle after
    the config's 10 steps, with the default setting of the OC the bench labels
    (C2: ST_TB_BM_RT_PR, C4: ST_CM_RT_PR) and the runner-up."""
    torch = _torch()
    C = si.CONFIGS[cfg]
    acc, c = si.config_stencil(C["stencil"])
    dims, dtype, steps = C["dims"], C["dtype"], C["steps"]
    x = torch.empty(dims, dtype=torch.float64, device="cuda")
    sm.fill_field(x, C["seed"])
    y = torch.empty_like(x)
    sm.Plan(dims, acc, c, dtype, sm.oc_from_name(oc)).run(x, y, steps)
    torch.cuda.synchronize()
    got = y.cpu().numpy()
    del y
    ref = oracle.sweep(x.cpu().numpy(), acc, c, steps, dtype=dtype)
    del x
    torch.cuda.empty_cache()
    assert _relerr(got, ref) <= TOL[dtype], oc


@pytest.mark.parametrize("oc, prm", [("base", None), ("TB_BM", None), ("ST_TB_BM_RT_PR", None)])
def test_graph_replay(gpu, monkeypatch, oc, prm):
    """Round 2: stencil_run replays a CUDA graph of its launch sequence from the
    second identical (in, out, workspace, steps) call on (api.cpp run_device).
    Every call -- eager, captured, replayed, after a key change -- must give the
    oracle's result, and every call must count the same kernel launches."""
    torch = _torch()
    monkeypatch.setenv("STENCIL_GRAPHS", "1")
    acc, c = si.config_stencil("random3d:1:0")
    dims = (20, 22, 68)
    u0 = si.make_field(dims, 5, "f64")
    p = sm.Plan(dims, acc, c, "f64", oc, prm)
    x = _to_dev(u0, "f64")
    y = torch.empty_like(x)
    z = torch.empty_like(x)
    refs = {s: oracle.sweep(u0, acc, c, s) for s in (3, 4)}
    counts = []
    for steps, out in ((3, y), (3, y), (3, y), (3, y), (4, y), (4, y), (4, y), (3, z), (3, z), (3, z), (3, y)):
        out.fill_(float("nan"))
        n0 = sm.launch_count()
        p.run(x, out, steps)
        torch.cuda.synchronize()
        counts.append((steps, sm.launch_count() - n0))
        assert _relerr(out.cpu().numpy(), refs[steps]) <= 1e-12, (oc, steps, len(counts))
    for s in (3, 4):
        assert len({n for st, n in counts if st == s}) == 1, counts


@pytest.mark.parametrize("stencil, oc", [("random2d:1:0", "TB_BM"), ("random2d:2:4", "TB_BM"),
                                         ("random2d:3:8", "TB_BM"), ("random2d:2:4", "TB_CM")])
def test_full_grid_n2_tiled_tb(gpu, stencil, oc):
    """Round 2: N2's whole 8192^2 fp64 grid after its 10 steps, element by element
    against the oracle, through the round-2 k_tiled TB path the bench labels for
    orders 1-2 (full-width 1 x 5 intermediate tiles, 2-column tiles for x-extent
    >= 3, 64 x 32 tiles) -- default settings, as the bench times them."""
    torch = _torch()
    C = si.CONFIGS["N2"]
    acc, c = si.config_stencil(stencil)
    dims, dtype, steps = C["dims"], C["dtype"], C["steps"]
    x = torch.empty(dims, dtype=torch.float64, device="cuda")
    sm.fill_field(x, C["seed"])
    y = torch.empty_like(x)
    sm.Plan(dims, acc, c, dtype, sm.oc_from_name(oc)).run(x, y, steps)
    torch.cuda.synchronize()
    got = y.cpu().numpy()
    del y
    ref = oracle.sweep(x.cpu().numpy(), acc, c, steps, dtype=dtype)
    del x
    torch.cuda.empty_cache()
    assert _relerr(got, ref) <= TOL[dtype], (stencil, oc)


@pytest.mark.parametrize("env, name, dims, dtype, oc", [
    ("STENCIL_NO_M8", "heat3d", (26, 70, 136), "f64", "ST_TB_BM_RT_PR"),
    ("STENCIL_TILED_FULL", "random2d:2:4", (200, 300), "f64", "TB_BM"),
    ("STENCIL_TILED_FULL", "random3d:2:5", (24, 40, 72), "f64", "TB_CM"),
    ("STENCIL_TILED_MVX", "star25", (20, 36, 72), "f32", "TB_BM"),
])
def test_round2_paths_bitwise_equal_to_round1(gpu, monkeypatch, env, name, dims, dtype, oc):
    """Round 2's kernel-path choices (8-row TB-RT setting, full-width and
    2-column k_tiled intermediate tiles) must not change a single bit of the
    result: every OC follows the canonical FMA order. Each pair is run with the
    switch that restores the round-1 path, 10 steps, and checked against the
    oracle too."""
    acc, c = si.config_stencil(name)
    u0 = si.make_field(dims, 13, dtype)
    ref = oracle.sweep(u0, acc, c, 10, dtype=dtype)
    outs = []
    for val in (None, "1" if env == "STENCIL_NO_M8" else ("0" if env == "STENCIL_TILED_FULL" else "1")):
        if val is None:
            monkeypatch.delenv(env, raising=False)
        else:
            monkeypatch.setenv(env, val)
        outs.append(_run(sm.Plan(dims, acc, c, dtype, oc), u0, dtype, 10))
    assert _relerr(outs[0], ref) <= TOL[dtype]
    assert np.array_equal(outs[0], outs[1])
