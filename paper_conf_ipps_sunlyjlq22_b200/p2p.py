"""Registration of the fused device-initiated halo transport.

One process per GPU: every rank publishes CUDA IPC handles of its registered
grids (in, out, workspace) and of its 16-byte flag buffer over
torch.distributed (any backend: only host bytes move), maps its neighbours'
(ranks +-1) into its address space and calls stencil_plan_set_p2p. Argument
marshalling only: the halo itself moves inside the edge kernels
(stencil_kernels.cuh, smart::Grid::peer_lo / peer_hi).
"""
from __future__ import annotations

from typing import List, Optional, Tuple

from .binding import P2PBuffers, Plan, ipc_close, ipc_handle, ipc_open


def new_flags(device) -> "torch.Tensor":
    """A zeroed 16-byte flag buffer (flags[0] written by rank-1, flags[1] by rank+1)."""
    import torch
    return torch.zeros(4, dtype=torch.int32, device=device)


class P2PLink:
    """Keeps the peer mappings of one registration alive; close() unmaps them."""

    def __init__(self, opened: List[Tuple[int, int]]):
        self._opened = opened

    def close(self) -> None:
        for ptr, off in self._opened:
            ipc_close(ptr, off)
        self._opened = []


def setup_p2p(plan: Plan, x, y, ws, flags, rank: int, world: int, group=None) -> P2PLink:
    """Collective: register `plan` (a slab of rank `rank`) with the P2P transport.

    x, y, ws: this rank's grids for stencil_run(plan, x, y, ...) and its
    workspace (plan.use_workspace(ws) is called here); flags: new_flags().
    """
    import torch
    import torch.distributed as dist

    torch.cuda.synchronize()                       # flags zeroed before anyone can signal
    mine = {"in": ipc_handle(x.data_ptr()), "out": ipc_handle(y.data_ptr()), "ws": ipc_handle(ws.data_ptr()),
            "flags": ipc_handle(flags.data_ptr()), "owned": int(plan.dims[0])}
    every: List[Optional[dict]] = [None] * world
    dist.all_gather_object(every, mine, group=group)
    opened: List[Tuple[int, int]] = []

    def peer(r: int) -> Optional[P2PBuffers]:
        if r < 0 or r >= world:
            return None
        ptrs = {}
        for key in ("in", "out", "ws", "flags"):
            h, off = every[r][key]
            ptrs[key] = ipc_open(h, off)
            opened.append((ptrs[key], off))
        return P2PBuffers(ptrs["in"], ptrs["out"], ptrs["ws"], ptrs["flags"], every[r]["owned"])

    selfb = P2PBuffers(x.data_ptr(), y.data_ptr(), ws.data_ptr(), flags.data_ptr(), int(plan.dims[0]))
    plan.set_p2p(rank, world, selfb, peer(rank - 1), peer(rank + 1))
    plan.use_workspace(ws)                         # sized for the slab (ghosts) after registration
    dist.barrier(group=group)                      # every rank registered before any run
    return P2PLink(opened)
