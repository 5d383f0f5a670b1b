"""B200-native StencilMART hot path (Sun et al., IPDPS'22).

The sweep of an arbitrary generated 2-D/3-D stencil under every optimization
combination (OC) of Table I, and the per-OC timing sweep that labels the best
OC. Compute lives in libstencilmart.so (C ABI: include/stencil.h); this package
is its thin ctypes binding.
"""
from .binding import (F32, F64, NUM_OC, OC_BM, OC_CM, OC_PR, OC_RT, OC_ST, OC_TB, Plan, StencilError,
                      P2PBuffers, embed_tensor, exported_symbols, ipc_close, ipc_handle, ipc_open, p2p_buffers, features, fill_field, fma_probe, gstencil_per_s, launch_count, lib,
                      link_loopback, nccl_unique_id, oc_analysis, oc_from_name, oc_list, oc_name, oc_valid, run_group,
                      sample_params, slab_halo, slab_range)

__all__ = ["F32", "F64", "NUM_OC", "OC_BM", "OC_CM", "OC_PR", "OC_RT", "OC_ST", "OC_TB", "P2PBuffers", "Plan",
           "StencilError", "ipc_close", "ipc_handle", "ipc_open", "p2p_buffers",
           "embed_tensor", "exported_symbols", "features", "fill_field", "fma_probe", "gstencil_per_s", "launch_count", "lib",
           "link_loopback", "nccl_unique_id", "oc_analysis", "oc_from_name", "oc_list", "oc_name", "oc_valid", "run_group",
           "sample_params", "slab_halo", "slab_range"]
