"""Thin ctypes binding of include/stencil.h (argument marshalling only).

Every step of the stencil sweep runs in libstencilmart.so (NVRTC-specialised
sm_100a kernels); PyTorch only supplies device memory, the CUDA stream and
(for multi-GPU) the process group used to broadcast the NCCL unique id.
There is no CPU fallback: if the library is missing or a call fails, an
exception is raised.
"""
from __future__ import annotations

import ctypes
import math
import os
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

from . import _build

F32, F64 = 0, 1
OC_ST, OC_BM, OC_CM, OC_RT, OC_PR, OC_TB = 1, 2, 4, 8, 16, 32
NUM_OC = 30
FAMILIES = ("naive", "tiled", "stream", "stream_tb")

_ERRORS = {
    -1: "E_INVAL", -2: "E_OC_INVALID", -3: "E_OC_INFEASIBLE", -4: "E_NOMEM",
    -5: "E_CUDA", -6: "E_NCCL", -7: "E_NVRTC", -8: "E_STATE",
}


class StencilError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{_ERRORS.get(code, code)}: {msg}")
        self.code = code
        self.name = _ERRORS.get(code, str(code))


class Params(ctypes.Structure):
    _fields_ = [("smem", ctypes.c_int32), ("bx", ctypes.c_int32), ("by", ctypes.c_int32),
                ("bz", ctypes.c_int32), ("vx", ctypes.c_int32), ("merge", ctypes.c_int32),
                ("stream_chunk", ctypes.c_int32), ("tb_steps", ctypes.c_int32),
                ("pr_stages", ctypes.c_int32), ("reserved", ctypes.c_int32 * 3)]

    def to_dict(self) -> Dict[str, int]:
        return {k: int(getattr(self, k)) for k, _ in self._fields_ if k != "reserved"}

    @classmethod
    def from_dict(cls, d: Optional[dict]) -> "Params":
        p = cls()
        p.smem = -1
        for k, v in (d or {}).items():
            setattr(p, k, int(v))
        return p


class PlanInfo(ctypes.Structure):
    _fields_ = [("ndim", ctypes.c_int32), ("order", ctypes.c_int32), ("nnz", ctypes.c_int32),
                ("dtype", ctypes.c_int32), ("ext", ctypes.c_int32 * 6), ("oc", ctypes.c_uint32),
                ("params", Params), ("kernel_family", ctypes.c_int32), ("smem_bytes", ctypes.c_int32),
                ("threads", ctypes.c_int32), ("regs", ctypes.c_int32), ("uses_tma", ctypes.c_int32),
                ("points", ctypes.c_int64), ("kernel_name", ctypes.c_char * 128),
                ("reg_split", ctypes.c_int32 * 2), ("xshift", ctypes.c_int32),
                ("host_chunks", ctypes.c_int32)]


class Features(ctypes.Structure):
    _fields_ = [("order", ctypes.c_int32), ("nnz", ctypes.c_int32), ("sparsity", ctypes.c_double),
                ("nnz_order", ctypes.c_int32 * 4), ("nnz_ratio", ctypes.c_double * 4)]


class SweepRow(ctypes.Structure):
    _fields_ = [("oc", ctypes.c_uint32), ("setting", ctypes.c_int32), ("params", Params),
                ("time_ms", ctypes.c_float), ("status", ctypes.c_int32)]


class P2PBuffers(ctypes.Structure):
    """stencil_p2p_buffers_t: a rank's registered grids + flag words (device addresses)."""
    _fields_ = [("in_", ctypes.c_void_p), ("out", ctypes.c_void_p), ("ws", ctypes.c_void_p),
                ("flags", ctypes.c_void_p), ("owned_planes", ctypes.c_int64)]


_lib = None

_SIGS = {
    "stencil_features": (ctypes.c_int, [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.POINTER(Features)]),
    "stencil_embed_tensor": (ctypes.c_int, [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p]),
    "stencil_sweep_rows": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(SweepRow), ctypes.c_int,
                                          ctypes.POINTER(ctypes.c_int)]),
    "stencil_oc_analysis": (ctypes.c_int, [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
                                           ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                           ctypes.c_void_p, ctypes.c_void_p]),
    "stencil_plan_set_p2p": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.POINTER(P2PBuffers),
                                            ctypes.POINTER(P2PBuffers), ctypes.POINTER(P2PBuffers)]),
    "stencil_ipc_get_handle": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.POINTER(ctypes.c_int64)]),
    "stencil_ipc_open_handle": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int64, ctypes.POINTER(ctypes.c_void_p)]),
    "stencil_ipc_close": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int64]),
    "stencil_plan_create": (ctypes.c_int, [ctypes.POINTER(ctypes.c_void_p), ctypes.c_int,
                                           ctypes.POINTER(ctypes.c_int64), ctypes.c_int, ctypes.c_void_p,
                                           ctypes.c_void_p, ctypes.c_int, ctypes.c_uint32,
                                           ctypes.POINTER(Params)]),
    "stencil_plan_destroy": (None, [ctypes.c_void_p]),
    "stencil_plan_set_stream": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "stencil_plan_workspace_bytes": (ctypes.c_size_t, [ctypes.c_void_p]),
    "stencil_plan_set_workspace": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t]),
    "stencil_plan_info": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(PlanInfo)]),
    "stencil_run": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int]),
    "stencil_run_host": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int]),
    "stencil_oc_sweep": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int,
                                        ctypes.c_int, ctypes.c_int, ctypes.c_uint64,
                                        ctypes.POINTER(ctypes.c_float), ctypes.POINTER(ctypes.c_uint32),
                                        ctypes.POINTER(Params), ctypes.POINTER(ctypes.c_uint32)]),
    "stencil_oc_valid": (ctypes.c_int, [ctypes.c_uint32]),
    "stencil_oc_list": (ctypes.c_int, [ctypes.POINTER(ctypes.c_uint32)]),
    "stencil_oc_name": (ctypes.c_char_p, [ctypes.c_uint32]),
    "stencil_sample_params": (ctypes.c_int, [ctypes.c_uint32, ctypes.c_int, ctypes.c_int, ctypes.c_uint64,
                                             ctypes.c_int, ctypes.POINTER(Params)]),
    "stencil_fill_field": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int, ctypes.c_int,
                                          ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64),
                                          ctypes.POINTER(ctypes.c_int64), ctypes.c_uint64, ctypes.c_int,
                                          ctypes.c_void_p]),
    "stencil_fma_probe": (ctypes.c_int, [ctypes.c_int, ctypes.c_int64, ctypes.c_int, ctypes.c_void_p,
                                         ctypes.c_void_p, ctypes.POINTER(ctypes.c_double)]),
    "stencil_nccl_unique_id": (ctypes.c_int, [ctypes.c_void_p]),
    "stencil_plan_set_comm": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int, ctypes.c_int]),
    "stencil_slab_range": (ctypes.c_int, [ctypes.c_int64, ctypes.c_int, ctypes.c_int,
                                          ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64)]),
    "stencil_plans_link_loopback": (ctypes.c_int, [ctypes.POINTER(ctypes.c_void_p), ctypes.c_int]),
    "stencil_plan_set_nccl_comm": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int, ctypes.c_int]),
    "stencil_plan_share_comm": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_void_p]),
    "stencil_run_group": (ctypes.c_int, [ctypes.POINTER(ctypes.c_void_p), ctypes.c_int,
                                         ctypes.POINTER(ctypes.c_void_p), ctypes.POINTER(ctypes.c_void_p),
                                         ctypes.c_int]),
    "stencil_plan_ghost_planes": (ctypes.c_int, [ctypes.c_void_p]),
    "stencil_slab_halo": (ctypes.c_int, [ctypes.c_int, ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                         ctypes.c_int, ctypes.POINTER(ctypes.c_int64)]),
    "stencil_plan_set_timing": (ctypes.c_int, [ctypes.c_void_p, ctypes.c_int]),
    "stencil_plan_kernel_time": (ctypes.c_int, [ctypes.c_void_p, ctypes.POINTER(ctypes.c_double),
                                                ctypes.POINTER(ctypes.c_int64)]),
    "stencil_last_error": (ctypes.c_char_p, []),
    "stencil_launch_count": (ctypes.c_uint64, []),
    "stencil_abi_version": (ctypes.c_int, []),
}


def exported_symbols() -> List[str]:
    return list(_SIGS)


def lib(build_if_missing: bool = False):
    """Load libstencilmart.so (raises if it is missing: no fallback)."""
    global _lib
    if _lib is None:
        if build_if_missing and _build.needs_build():
            _build.build()
        if not os.path.exists(_build.LIB):
            raise ImportError(f"{_build.LIB} not built; run __graft_entry__.build()")
        L = ctypes.CDLL(_build.LIB)
        for name, (res, args) in _SIGS.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _check(rc: int):
    if rc != 0:
        raise StencilError(rc, lib().stencil_last_error().decode(errors="replace"))


def _dtype_code(dtype) -> int:
    s = str(dtype)
    if s in ("f64", "float64", "torch.float64", "double"):
        return F64
    if s in ("f32", "float32", "torch.float32", "float"):
        return F32
    raise ValueError(f"unsupported dtype {dtype}")


# ------------------------------------------------------------------ OC lattice

def oc_list() -> List[int]:
    ids = (ctypes.c_uint32 * 64)()
    n = lib().stencil_oc_list(ids)
    return [int(ids[i]) for i in range(n)]


def oc_name(oc: int) -> Optional[str]:
    s = lib().stencil_oc_name(oc)
    return s.decode() if s else None


def oc_valid(oc: int) -> bool:
    return bool(lib().stencil_oc_valid(oc))


def oc_from_name(name: str) -> int:
    if name == "base":
        return 0
    bits = {"ST": OC_ST, "BM": OC_BM, "CM": OC_CM, "RT": OC_RT, "PR": OC_PR, "TB": OC_TB}
    m = 0
    for part in name.split("_"):
        m |= bits[part]
    return m


def sample_params(oc: int, ndim: int, dtype, seed: int, k: int) -> Dict[str, int]:
    p = Params()
    _check(lib().stencil_sample_params(oc, ndim, _dtype_code(dtype), seed, k, ctypes.byref(p)))
    return p.to_dict()


def launch_count() -> int:
    return int(lib().stencil_launch_count())


def slab_range(nz_global: int, rank: int, nranks: int) -> Tuple[int, int]:
    a, b = ctypes.c_int64(), ctypes.c_int64()
    _check(lib().stencil_slab_range(nz_global, rank, nranks, ctypes.byref(a), ctypes.byref(b)))
    return int(a.value), int(b.value)


def features(access: np.ndarray) -> Dict[str, float]:
    """Table II features of an access tensor, same keys as oracle.features."""
    acc = np.ascontiguousarray(access, dtype=np.uint8)
    order = (acc.shape[0] - 1) // 2
    f = Features()
    _check(lib().stencil_features(acc.ndim, order, acc.ctypes.data, ctypes.byref(f)))
    out: Dict[str, float] = {"order": f.order, "nnz": f.nnz, "sparsity": f.sparsity}
    for n in range(4):
        out[f"nnz_order{n + 1}"] = f.nnz_order[n]
        out[f"nnzRatio_order{n + 1}"] = f.nnz_ratio[n]
    return out


def embed_tensor(access: np.ndarray) -> np.ndarray:
    """The access tensor centred in the fixed 9^d tensor of Fig. 6."""
    acc = np.ascontiguousarray(access, dtype=np.uint8)
    out = np.zeros((9,) * acc.ndim, dtype=np.uint8)
    _check(lib().stencil_embed_tensor(acc.ndim, (acc.shape[0] - 1) // 2, acc.ctypes.data, out.ctypes.data))
    return out


def oc_analysis(times, n_classes: int = 5) -> Dict[str, object]:
    """OC analysis of a (stencil x OC) matrix of per-OC shortest times:
    Fig. 1 gap, Fig. 2 wins, Fig. 3 PCC matrix, the PCC merge into n_classes
    groups with their representatives, and each stencil's class (stencil_oc_analysis)."""
    t = np.ascontiguousarray(np.asarray(times, dtype=np.float64))
    if t.ndim != 2:
        raise ValueError("times must be [n_stencils][n_oc]")
    ns, k = t.shape
    gap = np.zeros(ns, dtype=np.float64)
    wins = np.zeros(k, dtype=np.int32)
    pcc = np.zeros((k, k), dtype=np.float64)
    group = np.zeros(k, dtype=np.int32)
    rep = np.zeros(max(n_classes, 1), dtype=np.int32)
    labels = np.zeros(ns, dtype=np.int32)
    _check(lib().stencil_oc_analysis(ns, k, t.ctypes.data, n_classes, gap.ctypes.data, wins.ctypes.data,
                                     pcc.ctypes.data, group.ctypes.data, rep.ctypes.data, labels.ctypes.data))
    return {"gap": gap, "wins": wins, "pcc": pcc, "group": group.tolist(),
            "representative": [int(r) for r in rep if r >= 0], "labels": labels.tolist()}


def slab_halo(ghost: int, n: int, zlo_g: int, zhi_g: int, rank: int, nranks: int) -> Dict[str, Tuple[int, int]]:
    """Halo plane ranges of one exchange: {'recv_lo': (begin, count), 'send_lo', 'send_hi', 'recv_hi'}."""
    out = (ctypes.c_int64 * 8)()
    _check(lib().stencil_slab_halo(ghost, n, zlo_g, zhi_g, rank, nranks, out))
    v = [int(x) for x in out]
    return {"recv_lo": (v[0], v[1]), "send_lo": (v[2], v[3]), "send_hi": (v[4], v[5]), "recv_hi": (v[6], v[7])}


def link_loopback(plans: Sequence["Plan"]) -> None:
    """Link plans as the z-slabs (rank order) of one grid on this device."""
    arr = (ctypes.c_void_p * len(plans))(*[p._h.value for p in plans])
    _check(lib().stencil_plans_link_loopback(arr, len(plans)))


def run_group(plans: Sequence["Plan"], ins, outs, steps: int, stream=None) -> None:
    L = lib()
    for p, t in zip(plans, ins):
        p._check_tensor(t)
        if steps >= 2:
            p._ensure_ws(t.device)
        _check(L.stencil_plan_set_stream(p._h, ctypes.c_void_p(_stream_ptr(stream))))
    hp = (ctypes.c_void_p * len(plans))(*[p._h.value for p in plans])
    hi = (ctypes.c_void_p * len(plans))(*[t.data_ptr() for t in ins])
    ho = (ctypes.c_void_p * len(plans))(*[t.data_ptr() for t in outs])
    _check(L.stencil_run_group(hp, len(plans), hi, ho, int(steps)))


def nccl_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * 128)()
    _check(lib().stencil_nccl_unique_id(buf))
    return bytes(buf)


def _stream_ptr(stream) -> int:
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return int(stream.cuda_stream)


def fill_field(t, seed: int, kind: int = 0, origin: Optional[Sequence[int]] = None,
               global_dims: Optional[Sequence[int]] = None, stream=None) -> None:
    """Device-side counter-based generator (same values as stencil_inputs.make_field)."""
    import torch
    assert t.is_cuda and t.is_contiguous()
    nd = t.dim()
    box = (ctypes.c_int64 * nd)(*t.shape)
    org = (ctypes.c_int64 * nd)(*(origin or [0] * nd))
    gd = (ctypes.c_int64 * nd)(*(global_dims or t.shape))
    dt = F64 if t.dtype == torch.float64 else F32
    _check(lib().stencil_fill_field(ctypes.c_void_p(t.data_ptr()), dt, nd, box, org, gd, seed, kind,
                                    ctypes.c_void_p(_stream_ptr(stream))))


def fma_probe(sink, iters: int, blocks_per_sm: int = 8, stream=None) -> float:
    """Enqueue one FMA-throughput probe launch (stencil_fma_probe) in the dtype
    of the device tensor `sink`; returns the launch's flops (time it with CUDA
    events on the same stream)."""
    import torch
    assert sink.is_cuda and sink.numel() >= 1
    fl = ctypes.c_double()
    dt = F64 if sink.dtype == torch.float64 else F32
    _check(lib().stencil_fma_probe(dt, int(iters), int(blocks_per_sm), ctypes.c_void_p(sink.data_ptr()),
                                   ctypes.c_void_p(_stream_ptr(stream)), ctypes.byref(fl)))
    return float(fl.value)


# ------------------------------------------------------------------------ plan

class Plan:
    """One stencil on one grid shape under one OC and parameter setting."""

    def __init__(self, dims: Sequence[int], access: np.ndarray, coeffs: np.ndarray, dtype="f64",
                 oc: int | str = 0, params: Optional[dict] = None):
        L = lib()
        if isinstance(oc, str):
            oc = oc_from_name(oc)
        self.dims = tuple(int(d) for d in dims)
        self.ndim = len(self.dims)
        acc = np.ascontiguousarray(access, dtype=np.uint8)
        cf = np.ascontiguousarray(coeffs, dtype=np.float64)
        self.order = (acc.shape[0] - 1) // 2
        if acc.shape != (2 * self.order + 1,) * self.ndim or cf.shape != acc.shape:
            raise ValueError("access/coeffs must have shape (2r+1,)*ndim")
        self.dtype = _dtype_code(dtype)
        self.oc = int(oc)
        self._h = ctypes.c_void_p()
        cdims = (ctypes.c_int64 * self.ndim)(*self.dims)
        p = Params.from_dict(params) if params is not None else None
        _check(L.stencil_plan_create(ctypes.byref(self._h), self.ndim, cdims, self.order,
                                     acc.ctypes.data, cf.ctypes.data, self.dtype, self.oc,
                                     ctypes.byref(p) if p is not None else None))
        self._ws = None

    # -- lifetime
    def close(self):
        if self._h:
            lib().stencil_plan_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # -- facts
    @property
    def info(self) -> dict:
        i = PlanInfo()
        _check(lib().stencil_plan_info(self._h, ctypes.byref(i)))
        return {
            "ndim": i.ndim, "order": i.order, "nnz": i.nnz, "dtype": "f64" if i.dtype == F64 else "f32",
            "ext": list(i.ext), "oc": i.oc, "oc_name": oc_name(i.oc), "params": i.params.to_dict(),
            "family": FAMILIES[i.kernel_family], "smem_bytes": i.smem_bytes, "threads": i.threads,
            "regs": i.regs, "uses_tma": bool(i.uses_tma), "points": int(i.points),
            "kernel_name": i.kernel_name.decode(),
            "reg_split": (i.reg_split[0], i.reg_split[1]),
            "xshift": bool(i.xshift),
            "host_chunks": i.host_chunks,
        }

    @property
    def torch_dtype(self):
        import torch
        return torch.float64 if self.dtype == F64 else torch.float32

    def workspace_bytes(self) -> int:
        return int(lib().stencil_plan_workspace_bytes(self._h))

    def _ensure_ws(self, device):
        import torch
        if self._ws is None:
            n = self.workspace_bytes() // (8 if self.dtype == F64 else 4)
            self._ws = torch.empty(n, dtype=self.torch_dtype, device=device)
            _check(lib().stencil_plan_set_workspace(self._h, ctypes.c_void_p(self._ws.data_ptr()),
                                                    self.workspace_bytes()))

    def use_workspace(self, t) -> None:
        """Use a caller-owned device tensor (>= workspace_bytes()) as the ping-pong
        workspace, e.g. one workspace shared by several plans of the same shape."""
        if t.numel() * t.element_size() < self.workspace_bytes():
            raise ValueError("workspace tensor too small")
        self._ws = t
        _check(lib().stencil_plan_set_workspace(self._h, ctypes.c_void_p(t.data_ptr()), self.workspace_bytes()))

    @property
    def ghost(self) -> int:
        """Ghost planes on each side of the slab (0 without a communicator)."""
        return int(lib().stencil_plan_ghost_planes(self._h))

    @property
    def array_shape(self) -> Tuple[int, ...]:
        """Shape of the device buffers: dims, plus 2*ghost planes along z for a slab."""
        g = self.ghost
        return (self.dims[0] + 2 * g,) + self.dims[1:]

    def _check_tensor(self, t):
        shape = self.array_shape
        if not (t.is_cuda and t.is_contiguous() and t.dtype == self.torch_dtype and tuple(t.shape) == shape):
            raise ValueError(f"expected a contiguous CUDA {self.torch_dtype} tensor of shape {shape}")

    # -- sweeps
    def run(self, inp, out, steps: int, stream=None) -> None:
        self._check_tensor(inp)
        self._check_tensor(out)
        if steps >= 2:
            self._ensure_ws(inp.device)
        L = lib()
        _check(L.stencil_plan_set_stream(self._h, ctypes.c_void_p(_stream_ptr(stream))))
        _check(L.stencil_run(self._h, ctypes.c_void_p(inp.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                             int(steps)))

    def _check_host(self, a, name):
        """A host buffer for stencil_run_host: C-contiguous, the plan's dtype and
        array_shape, exactly workspace_bytes() long (the C call copies that many
        bytes each way, so anything smaller would be overrun)."""
        shape = self.array_shape
        want = np.float64 if self.dtype == F64 else np.float32
        if hasattr(a, "data_ptr"):            # torch
            ok = (not a.is_cuda and a.is_contiguous() and a.dtype == self.torch_dtype and tuple(a.shape) == shape
                  and a.numel() * a.element_size() == self.workspace_bytes())
        else:
            a = np.asarray(a) if not isinstance(a, np.ndarray) else a
            ok = (a.flags.c_contiguous and a.dtype == want and tuple(a.shape) == shape
                  and a.nbytes == self.workspace_bytes())
        if not ok:
            raise ValueError(f"{name}: expected a C-contiguous host {want.__name__} buffer of shape {shape}")
        if name == "out" and not hasattr(a, "data_ptr") and not a.flags.writeable:
            raise ValueError("out: host buffer is read-only")

    def run_host(self, inp, out, steps: int, stream=None) -> None:
        """End to end: host buffers in and out (pinned torch tensors or numpy)."""
        self._check_host(inp, "in")
        self._check_host(out, "out")

        def ptr(a):
            return a.data_ptr() if hasattr(a, "data_ptr") else a.ctypes.data
        L = lib()
        _check(L.stencil_plan_set_stream(self._h, ctypes.c_void_p(_stream_ptr(stream))))
        _check(L.stencil_run_host(self._h, ctypes.c_void_p(ptr(inp)), ctypes.c_void_p(ptr(out)), int(steps)))

    def oc_sweep(self, inp, out, steps: int, settings_per_oc: int = 4, reps: int = 5, seed: int = 0,
                 stream=None) -> dict:
        self._check_tensor(inp)
        self._check_tensor(out)
        self._ensure_ws(inp.device)
        L = lib()
        _check(L.stencil_plan_set_stream(self._h, ctypes.c_void_p(_stream_ptr(stream))))
        times = (ctypes.c_float * NUM_OC)()
        ids = (ctypes.c_uint32 * NUM_OC)()
        bp = (Params * NUM_OC)()
        best = ctypes.c_uint32()
        _check(L.stencil_oc_sweep(self._h, ctypes.c_void_p(inp.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                  int(steps), int(settings_per_oc), int(reps), int(seed), times, ids, bp,
                                  ctypes.byref(best)))
        n = ctypes.c_int()
        _check(L.stencil_sweep_rows(self._h, None, 0, ctypes.byref(n)))
        rows = (SweepRow * max(n.value, 1))()
        _check(L.stencil_sweep_rows(self._h, rows, n.value, ctypes.byref(n)))
        return {
            "times_ms": [float(times[i]) for i in range(NUM_OC)],
            "oc_ids": [int(ids[i]) for i in range(NUM_OC)],
            "best_params": [bp[i].to_dict() for i in range(NUM_OC)],
            "best_oc": int(best.value),
            "rows": [{"oc": int(r.oc), "oc_name": oc_name(r.oc), "setting": int(r.setting),
                      "params": r.params.to_dict(), "time_ms": float(r.time_ms), "status": int(r.status)}
                     for r in rows[:n.value]],
        }

    def set_timing(self, enable: bool) -> None:
        _check(lib().stencil_plan_set_timing(self._h, int(bool(enable))))

    def kernel_time(self) -> Tuple[float, int]:
        """(summed device ms of the sweep-kernel launches since the last call, launches)."""
        ms, n = ctypes.c_double(), ctypes.c_int64()
        _check(lib().stencil_plan_kernel_time(self._h, ctypes.byref(ms), ctypes.byref(n)))
        return float(ms.value), int(n.value)

    def set_comm(self, uid: bytes, rank: int, nranks: int) -> None:
        """New NCCL communicator from a unique id (one communicator per id)."""
        buf = (ctypes.c_uint8 * 128).from_buffer_copy(uid)
        _check(lib().stencil_plan_set_comm(self._h, buf, rank, nranks))

    def set_nccl_comm(self, comm_ptr: int, rank: int, nranks: int) -> None:
        """Adopt an existing ncclComm_t (e.g. torch's: ProcessGroupNCCL._comm_ptr())."""
        _check(lib().stencil_plan_set_nccl_comm(self._h, ctypes.c_void_p(comm_ptr), rank, nranks))

    def set_p2p(self, rank: int, nranks: int, self_bufs: P2PBuffers, lo: Optional[P2PBuffers],
                hi: Optional[P2PBuffers]) -> None:
        """Fused device-initiated halo transport (stencil_plan_set_p2p): the edge
        kernels store the neighbours' ghost planes through peer memory."""
        self._p2p = (self_bufs, lo, hi)  # keep the structs alive
        _check(lib().stencil_plan_set_p2p(self._h, rank, nranks, ctypes.byref(self_bufs),
                                          ctypes.byref(lo) if lo is not None else None,
                                          ctypes.byref(hi) if hi is not None else None))

    def share_comm(self, other: "Plan") -> None:
        self._comm_src = other          # keep the owner alive
        _check(lib().stencil_plan_share_comm(self._h, other._h))


def ipc_handle(ptr: int) -> Tuple[bytes, int]:
    """CUDA IPC handle (64 bytes) of the allocation holding device address ptr, and ptr's offset in it."""
    h = (ctypes.c_uint8 * 64)()
    off = ctypes.c_int64()
    _check(lib().stencil_ipc_get_handle(ctypes.c_void_p(ptr), h, ctypes.byref(off)))
    return bytes(h), int(off.value)


def ipc_open(handle: bytes, offset: int) -> int:
    """Map a peer process's allocation; returns the device address of the same byte."""
    h = (ctypes.c_uint8 * 64).from_buffer_copy(handle)
    p = ctypes.c_void_p()
    _check(lib().stencil_ipc_open_handle(h, int(offset), ctypes.byref(p)))
    return int(p.value)


def ipc_close(ptr: int, offset: int) -> None:
    _check(lib().stencil_ipc_close(ctypes.c_void_p(ptr), int(offset)))


def p2p_buffers(inp: int, out: int, ws: int, flags: int, owned_planes: int) -> P2PBuffers:
    return P2PBuffers(inp, out, ws, flags, owned_planes)


def gstencil_per_s(points: int, steps: int, ms: float) -> float:
    return points * steps / (ms * 1e-3) / 1e9 if ms > 0 and math.isfinite(ms) else 0.0
