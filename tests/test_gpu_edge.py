"""GPU parity on the method's edge cases, every OC, 10 time steps.

The stencil definition (§I) and the access tensor (§IV-B) admit
patterns the config workloads never exercise: one-sided and asymmetric extents
(the per-axis halo lo/hi of every kernel's box, the TMA box origin, the slab
halo split), an extent smaller than the declared order (Table II "order: the
maximum extent", P:L178 -- the frame stays the declared width), no neighbours
along the streaming axis (NZ = 1), the centre alone, a centre coefficient of 0,
and mixed-sign coefficients. Each runs through all 30 Table I OCs at 10 steps
(the north-star bar) against the oracle:

* positive patterns, u0 in [1,2): pointwise relative error <= 1e-12 (fp64) /
  1e-5 (fp32), and every OC bitwise equal to OC base (canonical order, C-4);
* mixed-sign dyadic patterns on integer inputs: bitwise equal to the oracle
  (pin P7: every partial sum is exact, 10 + 4*T <= 53 in fp64, T <= 3 in fp32).

Grids are ragged against every tile, and both 16-byte-aligned rows (TMA staging)
and unaligned rows (cp.async staging of the streaming TB kernels) are covered.
"""
import concurrent.futures as cf
import os

import numpy as np
import pytest

import oracle
import paper_conf_ipps_sunlyjlq22_b200 as sm
import stencil_inputs as si

pytestmark = pytest.mark.gpu

TOL = {"f64": 1e-12, "f32": 1e-5}
MIXED = {"mixed3d", "mixed3d_r2", "mixed2d"}


def _plans(acc, c, dims, dtype, ocs, params=None):
    def mk(oc):
        return sm.Plan(dims, acc, c, dtype, oc, params(oc) if callable(params) else params)
    with cf.ThreadPoolExecutor(os.cpu_count() or 8) as ex:
        return dict(zip(ocs, ex.map(mk, ocs)))


def _run(plan, u0, dtype, steps):
    import torch
    x = torch.from_numpy(np.ascontiguousarray(u0)).cuda()
    y = torch.empty_like(x)
    plan.run(x, y, steps)
    torch.cuda.synchronize()
    return y.cpu().numpy()


def _relerr(got, ref):
    return float(np.max(np.abs(got.astype(np.float64) - ref) / np.maximum(np.abs(ref), 1e-300)))


def _cases():
    out = []
    for name in si.EDGE_3D:
        out.append((name, (37, 45, 70), "f64"))       # 560-byte rows: TMA
        out.append((name, (33, 38, 67), "f32"))       # 268-byte rows: cp.async staging
    for name in ("asym3d", "asym3d_lo"):
        out.append((name, (30, 41, 69), "f64"))       # unaligned fp64 rows
        out.append((name, (34, 39, 72), "f32"))       # aligned fp32 rows
    for name in si.EDGE_2D:
        out.append((name, (61, 83), "f64"))
        out.append((name, (70, 96), "f32"))
    out.append(("asym2d", (66, 96), "f64"))
    return out


@pytest.mark.parametrize("name,dims,dtype", _cases())
def test_edge_every_oc_10_steps(gpu, name, dims, dtype):
    acc, c = si.config_stencil("edge:" + name)
    mixed = name in MIXED
    steps = 3 if (mixed and dtype == "f32") else 10
    u0 = si.make_field(dims, 13, dtype, kind="int1023" if mixed else "uniform12")
    ref = oracle.sweep(u0, acc, c, steps, dtype=dtype)
    ocs = sm.oc_list()
    plans = _plans(acc, c, dims, dtype, ocs)       # every OC is feasible on these shapes
    base = None
    for oc in ocs:
        p = plans[oc]
        got = _run(p, u0, dtype, steps)
        if mixed:
            assert np.array_equal(got.astype(np.float64), ref), (sm.oc_name(oc), p.info["kernel_name"])
        else:
            err = _relerr(got, ref)
            assert err <= TOL[dtype], (sm.oc_name(oc), err, p.info["kernel_name"])
        if base is None:
            base = got
        else:
            assert np.array_equal(got, base), (sm.oc_name(oc), p.info["kernel_name"])


def test_unaligned_rows_stage_by_cp_async(gpu):
    """Streaming TB OCs on rows that no TMA tensor map can describe (fp64 rows of
    67 elements) stage their planes with cp.async; the info flag says so."""
    acc, c = si.config_stencil("edge:asym3d")
    dims = (30, 41, 67)
    for name in ("ST_TB", "ST_TB_BM_RT_PR", "ST_TB_CM_RT"):
        p = sm.Plan(dims, acc, c, "f64", sm.oc_from_name(name))
        assert p.info["uses_tma"] == 0, name
    p = sm.Plan((30, 41, 68), acc, c, "f64", sm.oc_from_name("ST_TB_RT"))
    assert p.info["uses_tma"] == 1


@pytest.mark.parametrize("name,dims,dtype", [("random3d:2:5", (31, 36, 50), "f64"),
                                             ("edge:asym3d", (29, 34, 45), "f32"),
                                             ("random2d:3:8", (70, 101), "f64")])
def test_label_pass_settings(gpu, name, dims, dtype):
    """Every setting the label pass times (stencil_oc_sweep: k = 0 the default,
    k >= 1 sampled by stencil_sample_params(seed, oc, k), P:L119 / P:L198) on all
    30 OCs, K = 3: a setting that is fast because it is wrong must not win a
    label. Infeasible settings (the paper's "crash") are skipped."""
    acc, c = si.config_stencil(name)
    steps, seed = 4, 7
    u0 = si.make_field(dims, 5, dtype)
    ref = oracle.sweep(u0, acc, c, steps, dtype=dtype)
    ran = 0
    for k in range(3):
        def prm(oc):
            return None if k == 0 else sm.sample_params(oc, len(dims), dtype, seed, k)

        def mk(oc):
            try:
                return sm.Plan(dims, acc, c, dtype, oc, prm(oc))
            except sm.StencilError as e:
                assert e.code == -3, (sm.oc_name(oc), k, str(e))
                return None
        with cf.ThreadPoolExecutor(os.cpu_count() or 8) as ex:
            plans = dict(zip(sm.oc_list(), ex.map(mk, sm.oc_list())))
        for oc, p in plans.items():
            if p is None:
                continue
            got = _run(p, u0, dtype, steps)
            assert _relerr(got, ref) <= TOL[dtype], (sm.oc_name(oc), k, p.info["params"])
            ran += 1
    assert ran >= 60
