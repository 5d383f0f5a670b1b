"""Python face of the oracle -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Never imported by the product package. Citations are PAPER.md line numbers.
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
from typing import Dict, List, Sequence, Tuple

import numpy as np

import stencil_inputs

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "stencil_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build_oracle(force: bool = False) -> str:
    """Compile stencil_oracle.c with gcc (-O2 -fopenmp -ffp-contract=off)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fPIC", "-shared",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build_oracle()
        lib = ctypes.CDLL(_LIB)
        lib.oracle_stencil_f64.restype = ctypes.c_int
        lib.oracle_stencil_f64.argtypes = [
            ctypes.c_int, ctypes.POINTER(ctypes.c_int64), ctypes.c_int,
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
            ctypes.c_int, ctypes.c_int]
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def sweep(u0: np.ndarray, access: np.ndarray, coeffs: np.ndarray, steps: int,
          dtype: str = "f64", nthreads: int = 0) -> np.ndarray:
    """u_T for the whole grid (frame rule C-1).

    fp32 mode (reading C-17 / SURVEY §8(c) c.1): the oracle consumes the
    fp32-rounded u_0 and fp32-rounded coefficients promoted to fp64, and never
    rounds to fp32 between steps. Returns float64.
    """
    ndim = u0.ndim
    order = (access.shape[0] - 1) // 2
    if access.shape != (2 * order + 1,) * ndim or coeffs.shape != access.shape:
        raise ValueError("access/coeffs must have shape (2r+1,)*ndim")
    if dtype == "f32":
        u = np.ascontiguousarray(u0.astype(np.float32).astype(np.float64))
        c = np.ascontiguousarray(coeffs.astype(np.float32).astype(np.float64))
    else:
        u = np.ascontiguousarray(u0, dtype=np.float64)
        c = np.ascontiguousarray(coeffs, dtype=np.float64)
    acc = np.ascontiguousarray(access, dtype=np.uint8)
    out = np.empty_like(u)
    dims = (ctypes.c_int64 * ndim)(*u.shape)
    rc = _load().oracle_stencil_f64(ndim, dims, order, acc.ctypes.data, c.ctypes.data,
                                    u.ctypes.data, out.ctypes.data, int(steps), int(nthreads))
    if rc != 0:
        raise RuntimeError(f"oracle_stencil_f64 failed rc={rc}")
    return out


def sweep_points(points: np.ndarray, global_dims: Sequence[int], seed: int, kind: str,
                 access: np.ndarray, coeffs: np.ndarray, steps: int, dtype: str = "f64") -> np.ndarray:
    """u_T at the given global points of a grid whose u_0 is the counter-based
    field ``stencil_inputs.make_field(global_dims, seed, dtype, kind)``.

    Each point is evaluated on its dependency cone: the sub-box of half-width
    steps*r around it (clipped to the grid), swept with :func:`sweep`. Values
    wrongly frozen at the sub-box faces reach at most (steps*r - 1) cells
    inward after ``steps`` steps, so the centre is exact; at global faces the
    sub-box frame is the global frame.
    """
    ndim = len(global_dims)
    order = (access.shape[0] - 1) // 2
    h = steps * order
    out = np.empty(len(points), dtype=np.float64)
    for i, p in enumerate(np.asarray(points, dtype=np.int64)):
        lo = [max(0, int(p[k]) - h) for k in range(ndim)]
        hi = [min(int(global_dims[k]), int(p[k]) + h + 1) for k in range(ndim)]
        box = stencil_inputs.make_field([b - a for a, b in zip(lo, hi)], seed, dtype, kind,
                                        origin=lo, global_dims=global_dims)
        # points within the global frame, or boxes too thin for an interior, are
        # handled by the same definition: sweep() copies frame cells.
        if any(b - a < 2 * order + 1 for a, b in zip(lo, hi)):
            # a thin box only happens at the global faces, where the point itself
            # lies in the frame and keeps u_0
            loc = tuple(int(p[k]) - lo[k] for k in range(ndim))
            out[i] = float(box[loc])
            continue
        res = sweep(box, access, coeffs, steps, dtype)
        out[i] = res[tuple(int(p[k]) - lo[k] for k in range(ndim))]
    return out


# --------------------------------------------------------------------------
# Table I: the OC lattice and the label
# --------------------------------------------------------------------------
OC_BITS: Dict[str, int] = {"ST": 1, "BM": 2, "CM": 4, "RT": 8, "PR": 16, "TB": 32}


def valid_ocs() -> List[int]:
    """All bitmasks allowed by Table I: BM and CM exclusive (rows 2-3), RT and
    PR only with ST (rows 4-5); ST and TB unconstrained (rows 1, 6)."""
    out = []
    for m in range(64):
        st, bm, cm, rt, pr = (bool(m & OC_BITS[k]) for k in ("ST", "BM", "CM", "RT", "PR"))
        if bm and cm:
            continue
        if (rt or pr) and not st:
            continue
        out.append(m)
    return out


def oc_name(mask: int) -> str:
    """'base' for the empty combination; otherwise abbreviations joined by '_'
    in the order ST, TB, BM, CM, RT, PR (so TB+CM is 'TB_CM' as at P:L93)."""
    parts = [k for k in ("ST", "TB", "BM", "CM", "RT", "PR") if mask & OC_BITS[k]]
    return "_".join(parts) if parts else "base"


def best_oc(times: Sequence[float], ids: Sequence[int]) -> int:
    """argmin over finite times; ties -> smallest OC id; all infinite -> -1."""
    best, best_t = -1, math.inf
    for t, i in sorted(zip(times, ids), key=lambda p: p[1]):
        if math.isfinite(t) and t < best_t:
            best, best_t = int(i), float(t)
    return best


# --------------------------------------------------------------------------
# Table II features, NEXT-1
# --------------------------------------------------------------------------

def features(access: np.ndarray, n_max: int = 4) -> Dict[str, float]:
    """order, nnz, sparsity, nnz_order-n, nnzRatio_order-n.

    Readings: the tensor is the fixed (2*n_max+1)^d embedding of
    P:L135, so sparsity = nnz / 9^d; "order-n neighbours" are the Chebyshev
    ring n (C-6), nnzRatio_order-n = nnz_order-n / |ring n|; the centre counts
    in nnz but in no ring.
    """
    d = access.ndim
    r = (access.shape[0] - 1) // 2
    nz = np.argwhere(access != 0) - r
    rings = np.max(np.abs(nz), axis=1) if len(nz) else np.zeros(0, dtype=int)
    out: Dict[str, float] = {
        "order": int(rings.max()) if len(rings) else 0,
        "nnz": int(len(nz)),
        "sparsity": len(nz) / float((2 * n_max + 1) ** d),
    }
    for n in range(1, n_max + 1):
        cnt = int(np.sum(rings == n))
        ring_size = (2 * n + 1) ** d - (2 * n - 1) ** d
        out[f"nnz_order{n}"] = cnt
        out[f"nnzRatio_order{n}"] = cnt / float(ring_size)
    return out
