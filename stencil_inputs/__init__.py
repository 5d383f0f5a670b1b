"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module holds NO arithmetic of the stencil method itself: it only draws
fields and stencils. Both `oracle/` (through the tests) and the product path
(through the tests and `bench.py`) consume what it produces; neither side imports
the other.

Contents
--------
* Counter-based field generator. Every value is a pure
  function of (seed, global linear index), so any sub-box of a huge grid can be
  regenerated independently. The CUDA runtime implements the *same* generator
  on the device (`stencil_fill_field` in `include/stencil.h`); a GPU test checks
  that the two agree bit for bit.
* Stencil builders: star / box shapes ("star, box and cross",
  orders 1-4) with the coefficient conventions of SURVEY §8(c) C-2.
* Algorithm 1, the random stencil generator (§IV-B),
  under the reading C-7 in DESIGN.md.

Layouts: grids are row-major, slowest dimension first (``[nz][ny][nx]``, 2-D
``[ny][nx]``). An access tensor of order r has shape ``(2r+1,)*ndim`` indexed
``[dz+r][dy+r][dx+r]`` ("the neighbor points accessed and the central
point are assigned a value of 1").
"""
from __future__ import annotations

import itertools
from typing import Dict, List, Sequence, Tuple

import numpy as np

# --------------------------------------------------------------------------
# counter-based generator (C-3)
# --------------------------------------------------------------------------
_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_SEEDMUL = np.uint64(0xD1B54A32D192ED03)

KINDS = ("uniform12", "int1023")


def mix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 output function applied to ``x + golden`` (wrapping uint64)."""
    with np.errstate(over="ignore"):
        z = (x + _GOLDEN).astype(np.uint64)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def hash_index(seed: int, gidx: np.ndarray) -> np.ndarray:
    """h(seed, g) = mix64((seed * 0xD1B54A32D192ED03) xor g)."""
    with np.errstate(over="ignore"):
        key = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) * _SEEDMUL
    return mix64(np.asarray(gidx, dtype=np.uint64) ^ key)


def values_from_hash(h: np.ndarray, dtype: str, kind: str) -> np.ndarray:
    """Map 64-bit hashes to field values.

    ``uniform12``: exactly uniform in [1, 2): fp64 takes 52 mantissa bits
    ``(h >> 12) | 0x3FF0...``, fp32 takes 23 bits ``(h >> 41) | 0x3F80...``.
    ``int1023``: integers in [-1023, 1023] (``(h >> 53) % 2047 - 1023``), the
    dyadic-exact pin P7 of SURVEY §8(c).
    """
    if kind == "uniform12":
        if dtype == "f64":
            bits = (h >> np.uint64(12)) | np.uint64(0x3FF0000000000000)
            return bits.view(np.float64)
        if dtype == "f32":
            bits = ((h >> np.uint64(41)) | np.uint64(0x3F800000)).astype(np.uint32)
            return bits.view(np.float32)
    elif kind == "int1023":
        v = ((h >> np.uint64(53)) % np.uint64(2047)).astype(np.int64) - 1023
        return v.astype(np.float64 if dtype == "f64" else np.float32)
    raise ValueError(f"bad dtype/kind {dtype}/{kind}")


def make_field(dims: Sequence[int], seed: int, dtype: str = "f64", kind: str = "uniform12",
               origin: Sequence[int] | None = None,
               global_dims: Sequence[int] | None = None) -> np.ndarray:
    """Field of shape ``dims`` whose element at local index i is
    ``value(h(seed, g))`` with g the row-major linear index of ``origin + i``
    inside ``global_dims`` (default: the box is the whole grid)."""
    dims = tuple(int(d) for d in dims)
    gdims = tuple(int(d) for d in (global_dims or dims))
    org = tuple(int(o) for o in (origin or (0,) * len(dims)))
    assert len(gdims) == len(dims) == len(org)
    strides = np.ones(len(dims), dtype=np.uint64)
    for k in range(len(dims) - 2, -1, -1):
        strides[k] = strides[k + 1] * np.uint64(gdims[k + 1])
    gidx = np.zeros(dims, dtype=np.uint64)
    for k, (n, o) in enumerate(zip(dims, org)):
        shape = [1] * len(dims)
        shape[k] = n
        gidx = gidx + (np.arange(o, o + n, dtype=np.uint64) * strides[k]).reshape(shape)
    return values_from_hash(hash_index(seed, gidx), dtype, kind)


# --------------------------------------------------------------------------
# stencil builders (P:L85 shapes; coefficients per C-2)
# --------------------------------------------------------------------------

def _empty(ndim: int, r: int):
    shape = (2 * r + 1,) * ndim
    return np.zeros(shape, dtype=np.uint8), np.zeros(shape, dtype=np.float64)


def star(ndim: int, r: int, centre: float, arm: Sequence[float]):
    """Star of order r: centre plus +-k along each axis, weight ``arm[k-1]``."""
    acc, c = _empty(ndim, r)
    ctr = (r,) * ndim
    acc[ctr] = 1
    c[ctr] = centre
    for ax in range(ndim):
        for k in range(1, r + 1):
            for s in (-1, 1):
                idx = list(ctr)
                idx[ax] += s * k
                acc[tuple(idx)] = 1
                c[tuple(idx)] = arm[k - 1]
    return acc, c


def box(ndim: int, r: int, centre: float, other: float):
    acc, c = _empty(ndim, r)
    acc[...] = 1
    c[...] = other
    c[(r,) * ndim] = centre
    return acc, c


def heat2d():
    """C1: 2-D 5-point heat, alpha = 1/8 -> centre 1/2, arms 1/8 (dyadic)."""
    return star(2, 1, 0.5, [0.125])


def heat3d():
    """C2: 3-D 7-point heat, alpha = 1/8 -> centre 1/4, arms 1/8 (dyadic)."""
    return star(3, 1, 0.25, [0.125])


def star25():
    """C3: order-4 3-D star, arm weights 1/16, 1/32, 1/64, 1/128, centre 19/64."""
    return star(3, 4, 19.0 / 64.0, [1 / 16, 1 / 32, 1 / 64, 1 / 128])


def box125():
    """C4: order-2 3-D box, 124 x 1/128 plus centre 4/128."""
    return box(3, 2, 4.0 / 128.0, 1.0 / 128.0)


# --------------------------------------------------------------------------
# Algorithm 1 under reading C-7
# --------------------------------------------------------------------------

def ring_index(offset: Sequence[int]) -> int:
    """Chebyshev ring of an offset (order = max extent, Table II)."""
    return max(abs(int(v)) for v in offset)


def _moore(p: Tuple[int, ...]) -> List[Tuple[int, ...]]:
    out = []
    for d in itertools.product((-1, 0, 1), repeat=len(p)):
        if any(d):
            out.append(tuple(a + b for a, b in zip(p, d)))
    return out


def random_stencil(ndim: int, order: int, seed: int, p: float = 0.5):
    """Algorithm 1: iteratively sample neighbours of the previous order's
    selected points, delete rings order-1 and order-2, append the set.

    Returns ``(access, npList)``; ``npList[k-1]`` is the set selected at order k.
    ``random()`` is an independent Bernoulli(p) draw per candidate, redrawn until
    at least one ring-``order`` point is kept (so the stencil order is exactly N).
    """
    if not (1 <= order <= 4) or ndim not in (2, 3):
        raise ValueError("order in 1..4, ndim in {2,3}")
    rng = np.random.Generator(np.random.PCG64(seed))
    centre = (0,) * ndim
    np_list: List[set] = []
    prev = {centre}
    for k in range(1, order + 1):
        cand = set()
        for q in sorted(prev):
            cand.update(_moore(q))
        if k >= 2:
            cand = {q for q in cand if ring_index(q) != k - 1}          # delete(neighbor_{k-1})
        if k > 2:
            cand = {q for q in cand if ring_index(q) != k - 2}          # delete(neighbor_{k-2})
        cand_sorted = sorted(cand)
        while True:
            keep = rng.random(len(cand_sorted)) < p
            sel = {q for q, kk in zip(cand_sorted, keep) if kk}
            if any(ring_index(q) == k for q in sel):
                break
        np_list.append(sel)
        prev = sel
    acc = np.zeros((2 * order + 1,) * ndim, dtype=np.uint8)
    acc[(order,) * ndim] = 1
    for s in np_list:
        for q in s:
            acc[tuple(v + order for v in q)] = 1
    return acc, np_list


def random_coeffs(access: np.ndarray, seed: int) -> np.ndarray:
    """C5 coefficients: U(0,1) on the accessed entries, normalised to sum 1."""
    rng = np.random.Generator(np.random.PCG64(seed ^ 0x5EED))
    c = np.where(access != 0, rng.random(access.shape), 0.0)
    return c / c.sum()


# --------------------------------------------------------------------------
# edge-case patterns (parity coverage of the method's degenerate cases)
# --------------------------------------------------------------------------

def pattern(ndim: int, order: int, weights: Dict[Tuple[int, ...], int], denom: int):
    """Access tensor + dyadic coefficients ``weights[o] / denom`` for the
    offsets ``o`` (slowest axis first). ``order`` is the DECLARED order (tensor
    size 2r+1, frame width r); the offsets may reach less far (Table II
    "order: the maximum extent", vs. the declared order of the
    tensor). The centre is always accessed; its weight may be 0."""
    acc, c = _empty(ndim, order)
    ctr = (order,) * ndim
    acc[ctr] = 1
    for o, w in weights.items():
        assert len(o) == ndim and max(abs(v) for v in o) <= order
        idx = tuple(order + v for v in o)
        acc[idx] = 1
        c[idx] = w / float(denom)
    return acc, c


# One-sided / asymmetric extents, extent < declared order, no neighbours along
# the streaming axis (NZ = 1), centre only, centre coefficient 0, mixed signs.
# Positive patterns sum to <= 1 (outputs stay in (0, 2) for u0 in [1, 2), so the
# pointwise relative error is well conditioned); the mixed-sign ones have
# sum |c| <= 1 with denominators 2^4 -> exact for integer inputs up to 10 steps
# in fp64 (10 + 4*10 <= 53, pin P7) and 3 steps in fp32 (10 + 4*3 <= 24).
EDGE_3D: Dict[str, Tuple[int, Dict[Tuple[int, int, int], int], int]] = {
    # zlo = 0, zhi = 2; ylo = 2, yhi = 1; xlo = 1, xhi = 3 (declared order 3)
    "asym3d": (3, {(0, 0, 0): 6, (1, 0, 0): 3, (2, 0, 0): 2, (0, 0, -1): 3, (0, 0, 1): 2, (0, 0, 2): 2,
                   (0, 0, 3): 1, (0, -2, 0): 2, (0, -1, 1): 3, (0, 1, 0): 2, (1, 1, 3): 1, (2, -2, -1): 1,
                   (1, -1, 2): 4}, 32),
    # mirror: zlo = 3, zhi = 0; ylo = 0, yhi = 2; xlo = 3, xhi = 0
    "asym3d_lo": (3, {(0, 0, 0): 8, (-1, 0, 0): 4, (-3, 0, 0): 2, (0, 0, -3): 2, (0, 0, -1): 4, (0, 2, 0): 4,
                      (0, 1, -2): 4, (-2, 1, -1): 2, (-1, 2, -3): 2}, 32),
    # extent 1 (the heat star) declared as order 3: frame width 3, halo 1
    "ext_lt_order3d": (3, {(0, 0, 0): 2, (1, 0, 0): 1, (-1, 0, 0): 1, (0, 1, 0): 1, (0, -1, 0): 1,
                           (0, 0, 1): 1, (0, 0, -1): 1}, 8),
    # no z neighbours (NZ = 1 plane in the streaming window): in-plane order 2
    "flat3d": (2, {(0, 0, 0): 4, (0, 0, 1): 2, (0, 0, -1): 2, (0, 1, 0): 2, (0, -1, 0): 2, (0, 1, 1): 1,
                   (0, -1, -1): 1, (0, 2, 0): 1, (0, 0, -2): 1}, 16),
    # z neighbours only (no in-plane halo)
    "zonly3d": (2, {(0, 0, 0): 4, (1, 0, 0): 1, (-1, 0, 0): 1, (2, 0, 0): 1, (-2, 0, 0): 1}, 8),
    # centre only; centre coefficient 0 (heat arms only)
    "centre3d": (1, {(0, 0, 0): 1}, 2),
    "zero_centre3d": (1, {(0, 0, 0): 0, (1, 0, 0): 1, (-1, 0, 0): 1, (0, 1, 0): 1, (0, -1, 0): 1,
                          (0, 0, 1): 1, (0, 0, -1): 1}, 8),
    # mixed signs, sum |k| = 16 = 2^4
    "mixed3d": (1, {(0, 0, 0): 5, (1, 0, 0): -2, (-1, 0, 0): 1, (0, 1, 0): 2, (0, -1, 1): -1, (0, 0, -1): 3,
                    (1, 1, 1): -1, (-1, -1, 0): 1}, 16),
    "mixed3d_r2": (2, {(0, 0, 0): 4, (2, 0, 0): -1, (-1, 0, 0): 2, (0, -2, 1): -2, (0, 1, 0): 1, (0, 0, 2): 3,
                       (1, 2, -2): -1, (-2, -1, -1): 2}, 16),
}
EDGE_2D: Dict[str, Tuple[int, Dict[Tuple[int, int], int], int]] = {
    # ylo = 0, yhi = 2; xlo = 1, xhi = 3
    "asym2d": (3, {(0, 0): 6, (1, 0): 3, (2, 0): 2, (0, -1): 3, (0, 1): 2, (0, 3): 2, (1, 2): 1, (2, -1): 1,
                   (1, -1): 2}, 22 + 10),
    "asym2d_lo": (2, {(0, 0): 4, (-2, 0): 2, (-1, -2): 1, (0, -1): 1}, 8),
    "ext_lt_order2d": (2, {(0, 0): 4, (1, 0): 1, (-1, 0): 1, (0, 1): 1, (0, -1): 1}, 8),
    # x neighbours only: NZ = 1 row in the streaming (y) window
    "row2d": (3, {(0, 0): 4, (0, -3): 1, (0, -1): 1, (0, 1): 1, (0, 2): 1}, 8),
    # y neighbours only (no x halo)
    "col2d": (2, {(0, 0): 4, (1, 0): 1, (-1, 0): 1, (2, 0): 1, (-2, 0): 1}, 8),
    "centre2d": (1, {(0, 0): 1}, 2),
    "zero_centre2d": (1, {(0, 0): 0, (1, 0): 1, (-1, 0): 1, (0, 1): 1, (0, -1): 1}, 4),
    "mixed2d": (2, {(0, 0): 5, (1, 0): -2, (-2, 0): 1, (0, 1): 2, (1, -2): -1, (0, -1): 3, (-1, 2): -2}, 16),
}


def edge_stencil(name: str):
    if name in EDGE_3D:
        r, w, d = EDGE_3D[name]
        return pattern(3, r, w, d)
    r, w, d = EDGE_2D[name]
    return pattern(2, r, w, d)


def config_stencil(name: str, seed: int = 0):
    """Named workloads of BASELINE.json configs."""
    if name.startswith("edge:"):
        return edge_stencil(name[5:])
    if name == "heat2d":
        return heat2d()
    if name == "heat3d":
        return heat3d()
    if name == "star25":
        return star25()
    if name == "box125":
        return box125()
    if name.startswith("random3d") or name.startswith("random2d"):
        # random{3,2}d:<order>:<seed>
        kind, order, s = name.split(":")
        acc, _ = random_stencil(3 if kind == "random3d" else 2, int(order), int(s))
        return acc, random_coeffs(acc, int(s))
    raise KeyError(name)


# --------------------------------------------------------------------------
# closed-form pin fields; inputs only, no stencil arithmetic
# --------------------------------------------------------------------------

def linear_field(dims: Sequence[int], a: Sequence[float], b: float) -> np.ndarray:
    grids = np.meshgrid(*[np.arange(n, dtype=np.float64) for n in dims], indexing="ij")
    return sum(ak * g for ak, g in zip(a, grids)) + b


def eigenmode_field(dims: Sequence[int], modes: Sequence[int]) -> np.ndarray:
    """prod_k sin(pi m_k i_k / (n_k - 1)); zero on the outer faces."""
    out = np.ones(tuple(dims), dtype=np.float64)
    for k, (n, m) in enumerate(zip(dims, modes)):
        shape = [1] * len(dims)
        shape[k] = n
        out = out * np.sin(np.pi * m * np.arange(n) / (n - 1)).reshape(shape)
    return out


def cosine_field(dims: Sequence[int], wave: Sequence[float], phase: float) -> np.ndarray:
    grids = np.meshgrid(*[np.arange(n, dtype=np.float64) for n in dims], indexing="ij")
    return np.cos(sum(k * g for k, g in zip(wave, grids)) + phase)


def dyadic_random_stencil(ndim: int, order: int, seed: int):
    """A random Alg.1 pattern with coefficients k_o / 2^m, integer k_o in
    [-3, 3] \\ {0} and m = ceil(log2 sum|k_o|) so that sum |c_o| <= 1 (pin P7:
    with integer |u_0| <= 1023 every partial sum is exact while 10 + m*T <= 53
    in fp64 or <= 24 in fp32). Returns ``(access, coeffs, m)``."""
    acc, _ = random_stencil(ndim, order, seed)
    rng = np.random.Generator(np.random.PCG64(seed + 77))
    nnz = int(acc.sum())
    ks = rng.integers(1, 4, size=nnz) * np.where(rng.random(nnz) < 0.3, -1, 1)
    m = int(np.ceil(np.log2(np.abs(ks).sum())))
    c = np.zeros(acc.shape)
    c[acc != 0] = ks / float(2 ** m)
    return acc, c, m


CONFIGS: Dict[str, dict] = {
    "C1": dict(ndim=2, dims=(256, 256), stencil="heat2d", dtype="f64", steps=10, seed=0xC0FFEE + 1),
    "C2": dict(ndim=3, dims=(512, 512, 512), stencil="heat3d", dtype="f64", steps=10, seed=0xC0FFEE + 2),
    "C3": dict(ndim=3, dims=(768, 768, 768), stencil="star25", dtype="f32", steps=10, seed=0xC0FFEE + 3),
    "C4": dict(ndim=3, dims=(512, 512, 512), stencil="box125", dtype="f64", steps=10, seed=0xC0FFEE + 4),
    "C5": dict(ndim=3, dims=(1024, 1024, 1024), stencil="random3d", dtype="f64", steps=4, seed=0xC0FFEE + 5),
    # NEXT-2: the paper's 2-D dataset size, 8192^2, random 2-D stencils
    "N2": dict(ndim=2, dims=(8192, 8192), stencil="random2d", dtype="f64", steps=10, seed=0xC0FFEE + 6),
}

# The stencils a multi-stencil workload sweeps: one Algorithm-1 stencil per
# order r = 1..4 (stencil seeds 0-15, order = 1 + seed/4;
# the bench takes the first seed of each order).
WORKLOAD_STENCILS: Dict[str, List[str]] = {
    "C5": [f"random3d:{r}:{4 * (r - 1)}" for r in range(1, 5)],
    "N2": [f"random2d:{r}:{4 * (r - 1)}" for r in range(1, 5)],
}
