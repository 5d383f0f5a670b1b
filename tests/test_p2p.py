"""Fused device-initiated halo (P2P transport) on one GPU.

The edge kernels store the neighbours' ghost planes through peer memory and
publish epochs in their flag words (include/stencil.h stencil_plan_set_p2p).
With one GPU the "peers" live on the same device:

* in one process: slab plans of one global grid on separate CUDA streams,
  registered with plain device pointers;
* across processes: two processes share cuda:0 and map each other's grids
  with CUDA IPC (the mapping a multi-GPU run uses), handles exchanged over a
  gloo process group.

Both must be bitwise equal to the single-domain run of the same OC (P10) and
within tolerance of the oracle.
"""
import os
import socket

import numpy as np
import pytest

import oracle
import stencil_inputs as si

torch = pytest.importorskip("torch")
import paper_conf_ipps_sunlyjlq22_b200 as sm  # noqa: E402
from paper_conf_ipps_sunlyjlq22_b200 import p2p  # noqa: E402

pytestmark = pytest.mark.gpu


def _slab_input(full, z0, z1, G, shape):
    x = torch.zeros(shape, dtype=full.dtype, device="cuda")
    a, b = max(0, z0 - G), min(full.shape[0], z1 + G)
    x[a - (z0 - G):b - (z0 - G)] = full[a:b]
    return x


@pytest.mark.parametrize("name,dtype,oc,steps,P,params", [
    ("heat3d", "f64", "base", 3, 2, None),
    ("heat3d", "f64", "ST_RT_PR", 5, 3, None),
    ("random3d:2:5", "f64", "TB", 5, 2, None),
    ("heat3d", "f64", "ST_TB_BM_RT_PR", 5, 2, None),
    ("random3d:3:1", "f32", "ST_TB_RT_PR", 4, 3, {"tb_steps": 3}),
    ("star25", "f32", "ST_BM_PR", 3, 2, None),
    ("box125", "f64", "ST_TB_CM", 4, 2, None),
    ("random3d:1:2", "f64", "ST_CM_RT", 6, 4, None),
    # one-sided / asymmetric z extents: the mirrored plane ranges differ per side
    ("edge:asym3d", "f64", "ST_TB_BM_RT_PR", 5, 3, None),       # zlo = 0, zhi = 2
    ("edge:asym3d_lo", "f64", "ST_RT_PR", 4, 2, None),          # zlo = 3, zhi = 0
    ("edge:zonly3d", "f32", "ST_TB_RT_PR", 5, 2, None),
    ("edge:asym3d", "f64", "TB_CM", 6, 2, {"tb_steps": 3})])
def test_p2p_in_process_bitwise(gpu, name, dtype, oc, steps, P, params):
    acc, c = si.config_stencil(name)
    gdims = (96, 36, 48) if P <= 3 else (160, 30, 40)
    tdt = torch.float64 if dtype == "f64" else torch.float32
    full = torch.empty(gdims, dtype=tdt, device="cuda")
    sm.fill_field(full, 23)
    ref_plan = sm.Plan(gdims, acc, c, dtype, oc, params)
    ref = torch.empty_like(full)
    ref_plan.run(full, ref, steps)
    torch.cuda.synchronize()

    plans, xs, ys, wss, flags, streams = [], [], [], [], [], []
    for k in range(P):
        z0, z1 = sm.slab_range(gdims[0], k, P)
        p = sm.Plan((z1 - z0,) + gdims[1:], acc, c, dtype, oc, params)
        plans.append(p)
    bufs = []
    for k, p in enumerate(plans):
        z0, z1 = sm.slab_range(gdims[0], k, P)
        G = 4 * ((acc.shape[0] - 1) // 2)              # stencil_plan_ghost_planes: 4 * order
        shape = (z1 - z0 + 2 * G,) + gdims[1:]
        xs.append(_slab_input(full, z0, z1, G, shape))
        ys.append(torch.empty(shape, dtype=tdt, device="cuda"))
        wss.append(torch.empty(shape, dtype=tdt, device="cuda"))
        flags.append(p2p.new_flags("cuda"))
        streams.append(torch.cuda.Stream())
        bufs.append(sm.P2PBuffers(xs[k].data_ptr(), ys[k].data_ptr(), wss[k].data_ptr(), flags[k].data_ptr(),
                                  z1 - z0))
    torch.cuda.synchronize()
    for k, p in enumerate(plans):
        p.set_p2p(k, P, bufs[k], bufs[k - 1] if k > 0 else None, bufs[k + 1] if k < P - 1 else None)
        assert p.ghost == 4 * ((acc.shape[0] - 1) // 2)
        p.use_workspace(wss[k])
    for k, p in enumerate(plans):      # each slab on its own stream; they wait on each other's flags
        p.run(xs[k], ys[k], steps, stream=streams[k])
    torch.cuda.synchronize()
    got = torch.cat([ys[k][p.ghost:p.ghost + p.dims[0]] for k, p in enumerate(plans)])
    assert torch.equal(got, ref), float((got - ref).abs().max())
    o = oracle.sweep(full.cpu().numpy(), acc, c, steps, dtype=dtype)
    tol = 1e-12 if dtype == "f64" else 1e-5
    assert float(np.max(np.abs(got.cpu().numpy() - o) / np.abs(o))) <= tol
    # a second run on the same registration (epochs continue) is identical
    for k, p in enumerate(plans):
        p.run(xs[k], ys[k], steps, stream=streams[k])
    torch.cuda.synchronize()
    got2 = torch.cat([ys[k][p.ghost:p.ghost + p.dims[0]] for k, p in enumerate(plans)])
    assert torch.equal(got2, ref)


def test_p2p_registration_errors(gpu):
    acc, c = si.config_stencil("heat3d")
    p = sm.Plan((20, 16, 16), acc, c, "f64", "ST_RT_PR")
    f = p2p.new_flags("cuda")
    x = torch.zeros((28, 16, 16), dtype=torch.float64, device="cuda")
    b = sm.P2PBuffers(x.data_ptr(), x.data_ptr(), x.data_ptr(), f.data_ptr(), 20)
    with pytest.raises(sm.StencilError):
        p.set_p2p(1, 2, b, None, None)                 # rank 1 needs its lower neighbour
    with pytest.raises(sm.StencilError):
        p.set_p2p(0, 2, sm.P2PBuffers(x.data_ptr(), x.data_ptr(), x.data_ptr(), f.data_ptr(), 19), None, b)
    p.set_p2p(0, 2, b, None, b)
    y = torch.zeros_like(x)
    with pytest.raises(sm.StencilError):               # unregistered buffers
        p.run(y, x, 1)
    with pytest.raises(sm.StencilError):               # label sweeps need NCCL
        p.oc_sweep(x, y, 1, settings_per_oc=1, reps=1)


# --------------------------------------------------------------- two processes, CUDA IPC
def _ipc_worker(rank, world, port, name, dtype, oc, steps, gdims, out_dir):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        acc, c = si.config_stencil(name)
        tdt = torch.float64 if dtype == "f64" else torch.float32
        full = torch.empty(gdims, dtype=tdt, device="cuda")
        sm.fill_field(full, 29)
        ref = torch.empty_like(full)
        sm.Plan(gdims, acc, c, dtype, oc).run(full, ref, steps)
        z0, z1 = sm.slab_range(gdims[0], rank, world)
        plan = sm.Plan((z1 - z0,) + gdims[1:], acc, c, dtype, oc)
        G = 4 * ((acc.shape[0] - 1) // 2)
        shape = (z1 - z0 + 2 * G,) + gdims[1:]
        x = _slab_input(full, z0, z1, G, shape)
        y = torch.empty(shape, dtype=tdt, device="cuda")
        ws = torch.empty(shape, dtype=tdt, device="cuda")
        flags = p2p.new_flags("cuda")
        link = p2p.setup_p2p(plan, x, y, ws, flags, rank, world)
        plan.run(x, y, steps)
        torch.cuda.synchronize()
        ok = torch.equal(y[G:G + z1 - z0], ref[z0:z1])
        dist.barrier()
        link.close()
        with open(os.path.join(out_dir, f"rank{rank}"), "w") as f:
            f.write("ok" if ok else "mismatch %g" % float((y[G:G + z1 - z0] - ref[z0:z1]).abs().max()))
    finally:
        dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


@pytest.mark.parametrize("name,dtype,oc,steps", [("heat3d", "f64", "ST_TB_BM_RT_PR", 5),
                                                  ("random3d:2:5", "f64", "ST_RT_PR", 4),
                                                  ("edge:asym3d", "f64", "ST_TB_CM_RT_PR", 5)])
def test_p2p_two_processes_ipc(gpu, tmp_path, name, dtype, oc, steps):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    port = _free_port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, name, dtype, oc, steps, (80, 34, 40), str(tmp_path)))
             for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0, p.exitcode
    for r in range(2):
        assert (tmp_path / f"rank{r}").read_text() == "ok"
