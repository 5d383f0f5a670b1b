"""Slab decomposition: host logic on CPU with gloo, and the full
C-ABI schedule on one GPU through the loopback transport.

* gloo, world size 2 and 3 (CPU): every rank evolves its slab with the oracle,
  exchanging halos with torch.distributed send/recv at the plane ranges the
  C ABI computes (stencil_slab_range, stencil_slab_halo); the gathered owned
  planes must equal the single-domain oracle bitwise (per-point arithmetic does
  not depend on the slab).
* loopback (GPU): P slabs of one grid as linked plans on one device; the edge /
  exchange / interior schedule of the NCCL path runs with cudaMemcpyAsync halos;
  the gathered result must equal the single-plan run bitwise (P10).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import paper_conf_ipps_sunlyjlq22_b200 as sm
import stencil_inputs as si


def _worker(rank, world, port, name, gdims, steps, T, result_q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        acc, c = si.config_stencil(name)
        r = (acc.shape[0] - 1) // 2
        offs = np.argwhere(acc) - r
        zlo, zhi = int(max(0, -offs[:, 0].min())), int(max(0, offs[:, 0].max()))
        G = 4 * r
        z0, z1 = sm.slab_range(gdims[0], rank, world)
        n = z1 - z0
        # local array: G ghost planes, n owned planes, G ghost planes
        arr = np.zeros((n + 2 * G,) + tuple(gdims[1:]))
        a, b = max(0, z0 - G), min(gdims[0], z1 + G)
        arr[a - (z0 - G):b - (z0 - G)] = si.make_field((b - a,) + tuple(gdims[1:]), 9, "f64",
                                                      origin=(a, 0, 0), global_dims=gdims)
        done = 0
        while done < steps:
            tl = min(T, steps - done)
            # oracle on the local array; the global frame only at the global faces
            lo = 0 if rank > 0 else G
            hi = n + 2 * G if rank < world - 1 else G + n
            arr[lo:hi] = oracle.sweep(np.ascontiguousarray(arr[lo:hi]), acc, c, tl)
            done += tl
            if done < steps:
                tn = min(T, steps - done)
                h = sm.slab_halo(G, n, tn * zlo, tn * zhi, rank, world)
                reqs = []
                bufs = {}
                for key, peer in (("send_lo", rank - 1), ("send_hi", rank + 1)):
                    s0, cnt = h[key]
                    if cnt:
                        reqs.append(dist.isend(torch.from_numpy(np.ascontiguousarray(arr[s0:s0 + cnt])), peer))
                for key, peer in (("recv_lo", rank - 1), ("recv_hi", rank + 1)):
                    s0, cnt = h[key]
                    if cnt:
                        bufs[key] = torch.empty((cnt,) + tuple(gdims[1:]), dtype=torch.float64)
                        reqs.append(dist.irecv(bufs[key], peer))
                for q in reqs:
                    q.wait()
                for key, t in bufs.items():
                    s0, cnt = h[key]
                    arr[s0:s0 + cnt] = t.numpy()
        own = torch.from_numpy(np.ascontiguousarray(arr[G:G + n]))
        parts = [torch.empty((sm.slab_range(gdims[0], k, world)[1] - sm.slab_range(gdims[0], k, world)[0],)
                             + tuple(gdims[1:]), dtype=torch.float64) for k in range(world)] if rank == 0 else None
        dist.gather(own, parts, dst=0)
        if rank == 0:
            result_q.put(np.concatenate([p.numpy() for p in parts]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,name,steps,T", [(2, "heat3d", 5, 1), (3, "random3d:2:5", 4, 2),
                                                (2, "random3d:1:3", 6, 4),
                                                # one-sided / asymmetric z extents (declared order 3)
                                                (2, "edge:asym3d", 5, 2), (3, "edge:asym3d_lo", 4, 1)])
def test_gloo_slab_exchange_matches_oracle(world, name, steps, T):
    gdims = (60, 12, 14) if not name.startswith("edge:") else (84, 12, 14)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    procs = [ctx.Process(target=_worker, args=(k, world, port, name, gdims, steps, T, q)) for k in range(world)]
    for p in procs:
        p.start()
    import queue
    import time
    t_end = time.time() + 300
    while True:          # fail fast when a rank dies instead of waiting out the timeout
        try:
            got = q.get(timeout=2)
            break
        except queue.Empty:
            dead = [p.exitcode for p in procs if p.exitcode not in (None, 0)]
            assert not dead and time.time() < t_end, f"gloo ranks failed: exit codes {dead}"
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    acc, c = si.config_stencil(name)
    ref = oracle.sweep(si.make_field(gdims, 9, "f64"), acc, c, steps)
    assert np.array_equal(got, ref)


def test_slab_halo_layout():
    h = sm.slab_halo(8, 100, 2, 3, 1, 3)
    assert h == {"recv_lo": (6, 2), "send_lo": (8, 3), "send_hi": (106, 2), "recv_hi": (108, 3)}
    h0 = sm.slab_halo(8, 100, 2, 3, 0, 3)
    assert h0["recv_lo"][1] == 0 and h0["send_lo"][1] == 0 and h0["send_hi"][1] == 2
    with pytest.raises(sm.StencilError):
        sm.slab_halo(8, 10, 2, 3, 0, 2)         # n < 2G


# ------------------------------------------------------------------ GPU loopback
def _loopback(name, gdims, dtype, oc, steps, P, params=None):
    acc, c = si.config_stencil(name)
    tdt = torch.float64 if dtype == "f64" else torch.float32
    full = torch.empty(gdims, dtype=tdt, device="cuda")
    sm.fill_field(full, 21)
    ref_plan = sm.Plan(gdims, acc, c, dtype, oc, params)
    ref = torch.empty_like(full)
    ref_plan.run(full, ref, steps)
    plans, ins, outs = [], [], []
    for k in range(P):
        z0, z1 = sm.slab_range(gdims[0], k, P)
        plans.append(sm.Plan((z1 - z0,) + tuple(gdims[1:]), acc, c, dtype, oc, params))
    sm.link_loopback(plans)
    for k, p in enumerate(plans):
        z0, z1 = sm.slab_range(gdims[0], k, P)
        G = p.ghost
        x = torch.zeros(p.array_shape, dtype=tdt, device="cuda")
        a, b = max(0, z0 - G), min(gdims[0], z1 + G)
        x[a - (z0 - G):b - (z0 - G)] = full[a:b]
        ins.append(x)
        outs.append(torch.empty_like(x))
    sm.run_group(plans, ins, outs, steps)
    torch.cuda.synchronize()
    got = torch.cat([outs[k][p.ghost:p.ghost + p.dims[0]] for k, p in enumerate(plans)])
    return got, ref, full


@pytest.mark.gpu
@pytest.mark.parametrize("name,dtype,oc,steps,P", [
    ("heat3d", "f64", "base", 3, 2), ("heat3d", "f64", "ST_RT_PR", 4, 3), ("random3d:2:5", "f64", "TB", 5, 2),
    ("random3d:3:1", "f32", "ST_TB_RT_PR", 5, 3), ("star25", "f32", "ST_BM_PR", 3, 2),
    ("box125", "f64", "ST_TB_CM", 4, 2),
    # one-sided / asymmetric z extents: halo counts differ per side (C-18)
    ("edge:asym3d", "f64", "ST_TB_RT_PR", 5, 3), ("edge:asym3d_lo", "f64", "ST_BM_RT_PR", 4, 2),
    ("edge:zonly3d", "f32", "TB", 5, 2), ("edge:flat3d", "f64", "ST_TB_CM", 4, 2)])
def test_loopback_slabs_bitwise(gpu, name, dtype, oc, steps, P):
    gdims = (100, 36, 48)
    got, ref, full = _loopback(name, gdims, dtype, oc, steps, P)
    assert torch.equal(got, ref), float((got - ref).abs().max())
    acc, c = si.config_stencil(name)
    o = oracle.sweep(full.cpu().numpy(), acc, c, steps, dtype=dtype)
    tol = 1e-12 if dtype == "f64" else 1e-5
    assert float(np.max(np.abs(got.cpu().numpy() - o) / np.abs(o))) <= tol
