"""Pins of the oracle against what the paper and mathematics fix (no GPU).

Each test names the SURVEY §8(c) pin it implements and the PAPER.md passage it
rests on. The oracle is never compared with itself: every expected value comes
from a library routine with a different evaluation order, a closed form, or an
independent brute-force loop.
"""
import itertools
import math

import numpy as np
import pytest
import torch

import oracle
import stencil_inputs as si


def _torch_step(u, coeffs):
    """Library reduction (P1): conv is cross-correlation sum_o c_o u[p+o]
    over the 'valid' region = the interior; the frame is copied (C-1)."""
    r = (coeffs.shape[0] - 1) // 2
    t = torch.from_numpy(np.ascontiguousarray(u, dtype=np.float64))[None, None]
    w = torch.from_numpy(np.ascontiguousarray(coeffs, dtype=np.float64))[None, None]
    conv = torch.nn.functional.conv3d if u.ndim == 3 else torch.nn.functional.conv2d
    inner = conv(t, w)[0, 0].numpy()
    out = u.copy()
    sl = tuple(slice(r, n - r) for n in u.shape)
    out[sl] = inner
    return out


def _interior(shape, h):
    return tuple(slice(h, n - h) for n in shape)


# ---------------------------------------------------------------- P1
@pytest.mark.parametrize("ndim,order,seed", [(3, 1, 1), (3, 2, 5), (3, 3, 9), (2, 4, 3), (2, 1, 4)])
def test_p1_library_conv(ndim, order, seed):
    acc, _ = si.random_stencil(ndim, order, seed)
    c = si.random_coeffs(acc, seed)
    dims = (19, 23, 21) if ndim == 3 else (37, 41)
    u = si.make_field(dims, seed, "f64")
    got = oracle.sweep(u, acc, c, 1)
    ref = _torch_step(u, c)
    assert np.max(np.abs(got - ref)) <= 1e-15 * acc.sum()


# ---------------------------------------------------------------- P2
def test_p2_constant_field():
    acc, c, m = si.dyadic_random_stencil(3, 2, 11)
    s = c.sum()
    assert s != 1.0
    val = 3.0
    u = np.full((24, 20, 22), val)
    for T in (1, 2, 3):
        got = oracle.sweep(u, acc, c, T)
        h = 2 * T
        assert np.all(got[_interior(u.shape, h)] == (s ** T) * val)
    # frame untouched
    got = oracle.sweep(u, acc, c, 2)
    assert np.all(got[0] == val) and np.all(got[:, :, -1] == val)


# ---------------------------------------------------------------- P3
def test_p3_linear_field_fixed_point():
    rng = np.random.default_rng(0)
    r = 2
    k = rng.integers(1, 5, size=(2 * r + 1,) * 3)
    k = k + k[::-1, ::-1, ::-1]                       # symmetric c_o = c_{-o}
    acc = np.ones_like(k, dtype=np.uint8)
    c = k / float(k.sum())
    # make the coefficient sum dyadic-exact: scale to a power of two
    m = int(math.ceil(math.log2(k.sum())))
    c = k / float(2 ** m)
    c[(r, r, r)] += 1.0 - c.sum()                      # sum exactly 1, still dyadic
    assert c.sum() == 1.0
    u = si.linear_field((16, 18, 20), (3.0, -2.0, 5.0), 7.0)
    got = oracle.sweep(u, acc, c, 4)
    assert np.max(np.abs(got - u)) == 0.0


# ---------------------------------------------------------------- P4
def test_p4_heat_eigenmode():
    acc, c = si.heat3d()
    dims, modes, T = (34, 30, 26), (1, 2, 3), 10
    u0 = si.eigenmode_field(dims, modes)
    alpha = 0.125
    lam = 1.0 - 4 * alpha * sum(math.sin(math.pi * m / (2 * (n - 1))) ** 2 for m, n in zip(modes, dims))
    got = oracle.sweep(u0, acc, c, T)
    err = np.max(np.abs(got - lam ** T * u0)) / np.max(np.abs(u0))
    assert err < 1e-14


# ---------------------------------------------------------------- P5
@pytest.mark.parametrize("ndim,order,seed,T", [(3, 2, 21, 3), (3, 1, 8, 4), (2, 3, 2, 2), (3, 4, 6, 1)])
def test_p5_fourier_symbol(ndim, order, seed, T):
    acc, _ = si.random_stencil(ndim, order, seed)
    c = si.random_coeffs(acc, seed)
    dims = (40,) * ndim if order < 4 else (30,) * ndim
    wave = [0.31, -0.47, 0.73][:ndim]
    phase = 0.2
    u0 = si.cosine_field(dims, wave, phase)
    offs = np.argwhere(acc != 0) - order
    sigma = sum(c[tuple(o + order)] * np.exp(1j * np.dot(wave, o)) for o in offs)
    grids = np.meshgrid(*[np.arange(n) for n in dims], indexing="ij")
    kp = sum(w * g for w, g in zip(wave, grids)) + phase
    expect = np.real(sigma ** T * np.exp(1j * kp))
    got = oracle.sweep(u0, acc, c, T)
    sl = _interior(dims, order * T)
    assert np.max(np.abs(got[sl] - expect[sl])) < 1e-14


# ---------------------------------------------------------------- P6
def test_p6_time_composition():
    from scipy.signal import convolve
    acc, _ = si.random_stencil(3, 2, 31)
    c = si.random_coeffs(acc, 31)
    T = 3
    cT = c
    for _ in range(T - 1):
        cT = convolve(cT, c, mode="full")          # C^{*T}, order T*r
    accT = (np.abs(cT) > 0).astype(np.uint8)
    cT = np.where(accT > 0, cT, 0.0)
    accT[(T * 2,) * 3] = 1
    u = si.make_field((30, 28, 26), 4, "f64")
    got = oracle.sweep(u, acc, c, T)
    one = oracle.sweep(u, accT, cT, 1)
    sl = _interior(u.shape, 2 * T)
    # rounding bound: up to 13^3 products per point, each within eps of exact
    assert np.max(np.abs(got[sl] - one[sl])) < accT.sum() * 2.3e-16 * 2


# ---------------------------------------------------------------- P7
@pytest.mark.parametrize("name,T", [("heat3d", 10), ("box125", 6), ("heat2d", 10)])
def test_p7_dyadic_bitwise_vs_library(name, T):
    acc, c = si.config_stencil(name)
    dims = (20, 22, 24) if acc.ndim == 3 else (40, 36)
    u = si.make_field(dims, 7, "f64", kind="int1023")
    got = oracle.sweep(u, acc, c, T)
    ref = u.copy()
    for _ in range(T):
        ref = _torch_step(ref, c)
    assert np.array_equal(got, ref)


def test_p7_dyadic_random_bitwise():
    acc, c, m = si.dyadic_random_stencil(3, 3, 13)
    T = (53 - 10) // m
    assert T >= 1
    u = si.make_field((21, 19, 23), 2, "f64", kind="int1023")
    got = oracle.sweep(u, acc, c, T)
    ref = u.copy()
    for _ in range(T):
        ref = _torch_step(ref, c)
    assert np.array_equal(got, ref)


def test_p7_fp32_mode_star25():
    """C3 fp32, m = 7: exact to T = 2; fp32 oracle == fp64 oracle bitwise."""
    acc, c = si.star25()
    u = si.make_field((20, 20, 20), 3, "f32", kind="int1023")
    got32 = oracle.sweep(u, acc, c, 2, dtype="f32")
    got64 = oracle.sweep(u.astype(np.float64), acc, c, 2)
    assert np.array_equal(got32, got64)


# ---------------------------------------------------------------- P8
def _brute(u, acc, c, T):
    """Per-point brute force over the DENSE tensor (not a compacted list)."""
    r = (acc.shape[0] - 1) // 2
    d = u.ndim
    cur = u.copy()
    for _ in range(T):
        nxt = cur.copy()
        for p in itertools.product(*[range(r, n - r) for n in u.shape]):
            s = 0.0
            for o in itertools.product(range(-r, r + 1), repeat=d):
                if acc[tuple(v + r for v in o)]:
                    s += c[tuple(v + r for v in o)] * cur[tuple(a + b for a, b in zip(p, o))]
            nxt[p] = s
        cur = nxt
    return cur


@pytest.mark.parametrize("order,n", [(1, 8), (2, 8), (3, 8), (4, 12)])
def test_p8_brute_force(order, n):
    acc, _ = si.random_stencil(3, order, 40 + order)
    c = si.random_coeffs(acc, 40 + order)
    u = si.make_field((n, n, n), order, "f64")
    T = 2 if order < 4 else 1
    got = oracle.sweep(u, acc, c, T)
    ref = _brute(u, acc, c, T)
    assert np.max(np.abs(got - ref)) < 1e-15 * 4


def test_p8_brute_force_2d():
    acc, _ = si.random_stencil(2, 2, 3)
    c = si.random_coeffs(acc, 3)
    u = si.make_field((11, 13), 1, "f64")
    got = oracle.sweep(u, acc, c, 3)
    assert np.max(np.abs(got - _brute(u, acc, c, 3))) < 1e-15 * 4


# ---------------------------------------------------------------- P11
def test_p11_linearity_translation():
    acc, _ = si.random_stencil(3, 2, 17)
    c = si.random_coeffs(acc, 17)
    u = si.make_field((22, 22, 22), 1, "f64")
    v = si.make_field((22, 22, 22), 2, "f64")
    a, b = 0.5, -2.0
    lhs = oracle.sweep(a * u + b * v, acc, c, 2)
    rhs = a * oracle.sweep(u, acc, c, 2) + b * oracle.sweep(v, acc, c, 2)
    assert np.max(np.abs(lhs - rhs)) < 1e-13
    # translation: shifting the input shifts the halo-free interior
    us = np.roll(u, (1, -2, 3), axis=(0, 1, 2))
    s0 = oracle.sweep(u, acc, c, 1)
    s1 = oracle.sweep(us, acc, c, 1)
    sl = _interior(u.shape, 6)
    assert np.array_equal(np.roll(s0, (1, -2, 3), axis=(0, 1, 2))[sl], s1[sl])


# ---------------------------------------------------------------- edge cases
def test_steps_zero_and_frame_only():
    acc, c = si.heat3d()
    u = si.make_field((5, 6, 7), 3, "f64")
    assert np.array_equal(oracle.sweep(u, acc, c, 0), u)
    tiny = si.make_field((2, 9, 9), 3, "f64")          # no interior along z
    assert np.array_equal(oracle.sweep(tiny, acc, c, 3), tiny)


def test_sweep_points_matches_full():
    acc, _ = si.random_stencil(3, 2, 55)
    c = si.random_coeffs(acc, 55)
    dims, seed, T = (26, 30, 28), 99, 3
    full = oracle.sweep(si.make_field(dims, seed, "f64"), acc, c, T)
    rng = np.random.default_rng(1)
    pts = np.stack([rng.integers(0, n, size=40) for n in dims], axis=1)
    pts = np.concatenate([pts, [[0, 0, 0], [2, 5, 27], [25, 29, 27], [6, 6, 6], [13, 2, 14]]])
    got = oracle.sweep_points(pts, dims, seed, "uniform12", acc, c, T)
    assert np.array_equal(got, full[tuple(pts.T)])


def test_fp32_mode_rounds_inputs_once():
    acc, c = si.config_stencil("random3d:3:4")
    u = si.make_field((18, 18, 18), 3, "f64")
    got = oracle.sweep(u, acc, c, 2, dtype="f32")
    ref = oracle.sweep(u.astype(np.float32).astype(np.float64), acc,
                       c.astype(np.float32).astype(np.float64), 2)
    assert np.array_equal(got, ref)


# ---------------------------------------------------------------- Table I
def test_table1_lattice():
    ids = oracle.valid_ocs()
    assert len(ids) == 30
    B = oracle.OC_BITS
    no_st = [m for m in ids if not m & B["ST"]]
    assert len(no_st) == 6 and len(ids) - len(no_st) == 24
    assert sorted(oracle.oc_name(m) for m in no_st) == sorted(
        ["base", "BM", "CM", "TB", "TB_BM", "TB_CM"])     # P:L93 names TB, TB_CM, TB_BM
    assert B["ST"] | B["RT"] in ids
    assert B["RT"] not in ids and B["PR"] | B["TB"] not in ids
    assert B["BM"] | B["CM"] not in ids and B["ST"] | B["BM"] | B["CM"] not in ids
    assert 63 not in ids and B["ST"] | B["BM"] | B["RT"] | B["PR"] | B["TB"] in ids


def test_best_oc_label():
    inf = math.inf
    assert oracle.best_oc([3.0, 1.0, 2.0], [0, 1, 3]) == 1
    assert oracle.best_oc([1.0, 1.0], [5, 2]) == 2              # tie -> smallest id
    assert oracle.best_oc([inf, 4.0, inf], [0, 1, 2]) == 1      # infeasible never best
    assert oracle.best_oc([inf, inf], [0, 1]) == -1


# ---------------------------------------------------------------- Table II
@pytest.mark.parametrize("d,r", [(2, 1), (2, 4), (3, 1), (3, 2), (3, 4)])
def test_table2_star_box(d, r):
    acc_s, _ = si.star(d, r, 1.0, [1.0] * r)
    f = oracle.features(acc_s)
    assert f["order"] == r and f["nnz"] == 2 * d * r + 1
    for k in range(1, r + 1):
        assert f[f"nnz_order{k}"] == 2 * d
    acc_b, _ = si.box(d, r, 1.0, 1.0)
    f = oracle.features(acc_b)
    assert f["nnz"] == (2 * r + 1) ** d
    assert f["sparsity"] == (2 * r + 1) ** d / 9.0 ** d
    for k in range(1, r + 1):
        assert f[f"nnz_order{k}"] == (2 * k + 1) ** d - (2 * k - 1) ** d
        assert f[f"nnzRatio_order{k}"] == 1.0
