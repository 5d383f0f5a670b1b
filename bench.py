#!/usr/bin/env python
"""bench.py -- GStencil/s and % of HBM roofline per OC on B200 (BASELINE.json metric).

Default workload ("C5", BASELINE.json configs[4]): the configuration the metric
is quoted on ("... per OC at 1/2/4/8 B200") and the largest per-GPU one -- four
random Algorithm-1 3-D stencils, one per order r = 1..4, 1024^3 fp64 per GPU,
4 time steps each, every OC of Table I swept per stencil, z-slabs with the halo
exchange at N > 1 (weak scaling). `--config C1..C4, N2` select the others.

What one run does (one process per GPU: torchrun, or `--gpus N` spawns the N
ranks itself):
  1. label pass: stencil_oc_sweep over the 30 OCs with the
     library's seeded settings; its per-OC times give "per_oc" (GStencil/s and
     HBM fraction of every OC) and the label (best OC + its setting);
  2. W warm-up steps, then K timed steps of the production path: one timed
     step = stencil_run of the config's 10 time steps with the labelled OC,
     inputs resident in HBM (1 GiB per grid >> 126 MB L2, so no flush is
     needed), bracketed by barrier + synchronize, CUDA events on the plan's
     stream, max over ranks;
  3. roofline of the dominant kernel (the labelled OC's sweep kernel): bytes a
     launch must move (read + write the grid once: 16 B / point in fp64, for
     every fused step count) / its average launch duration, from CUDA events
     around each launch over the timed region -- or, for FMA-bound stencils,
     flops / time against the FMA peak measured in the same run
     (stencil_fma_probe, `fma_peak`);
  4. e2e: the same metric through stencil_run_host (pinned host buffers in,
     H2D + 10 steps + D2H inside the timed region);
  5. cpu_baseline: the oracle (oracle/, plain C loops, OpenMP) on a bounded
     sample of the same workload on this host's cores (rank 0, N = 1 only).
`--impl reference` times only the oracle (the "reference arm" of this tier).
Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "GStencil/s and % of HBM roofline per OC at 1/2/4/8 B200"
L2_BYTES = 126 * 2**20
HBM_SPEC_GBS = 8000.0


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured"
    return 6650.0, "fallback"


WORKLOADS = {
    "C2": "C2: 3-D 7-point heat star (order 1), 512^3 fp64 per GPU, 10 time steps, all 30 OCs swept, best OC timed",
    "C3": "C3: 3-D 25-point star (order 4), 768^3 fp32 per GPU, 10 time steps, ST/RT family swept, best OC timed",
    "C4": "C4: 3-D 125-point box (order 2), 512^3 fp64 per GPU, 10 time steps, TB vs tiling family swept",
    "C1": "C1: 2-D 5-point heat star (order 1), 256^2 fp64, 10 time steps, naive OC",
    "C5": ("C5: random Algorithm-1 3-D stencils, one per order 1..4, 1024^3 fp64 per GPU, 4 time steps each, "
           "all 30 OCs swept per stencil, best OC per stencil timed"),
    "N2": ("N2 (NEXT-2): random Algorithm-1 2-D stencils, one per order 1..4, 8192^2 fp64 per GPU, 10 time "
           "steps each, all 30 OCs swept per stencil (streaming along y), best OC per stencil timed"),
}


def _free_port() -> int:
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _env_rank():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


class ClockSampler:
    """NVML SM clock + throttle reasons sampled during the timed region."""

    def __init__(self, index: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        self._t = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        nv = self.nv
        names = {
            "hw_slowdown": getattr(nv, "nvmlClocksEventReasonHwSlowdown", 0x8),
            "hw_thermal_slowdown": getattr(nv, "nvmlClocksEventReasonHwThermalSlowdown", 0x40),
            "sw_thermal_slowdown": getattr(nv, "nvmlClocksEventReasonSwThermalSlowdown", 0x20),
            "sw_power_cap": getattr(nv, "nvmlClocksEventReasonSwPowerCap", 0x4),
            "hw_power_brake_slowdown": getattr(nv, "nvmlClocksEventReasonHwPowerBrakeSlowdown", 0x80),
        }
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for k, bit in names.items():
                    if r & bit:
                        self.reasons.add(k)
            except Exception:
                pass
            self._stop.wait(0.005)

    def __enter__(self):
        if self.nv:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def result(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": len(self.samples)}


def _config(name: str):
    import stencil_inputs as si
    C = dict(si.CONFIGS[name])
    acc, c = si.config_stencil(C["stencil"] if name not in si.WORKLOAD_STENCILS else si.WORKLOAD_STENCILS[name][0])
    return C, acc, c


def _items(name: str):
    """The stencils one bench step sweeps: one for C1-C4, one per order r = 1..4
    for the multi-stencil workloads (C5 3-D, N2 2-D)."""
    import stencil_inputs as si
    names = si.WORKLOAD_STENCILS.get(name) or [si.CONFIGS[name]["stencil"]]
    out = []
    for sname in names:
        acc, c = si.config_stencil(sname)
        out.append({"stencil": sname, "acc": acc, "c": c})
    return out


def _ocs_for(name: str, sm):
    if name == "C3":
        return [o for o in sm.oc_list() if o & sm.OC_ST and not o & sm.OC_TB]
    if name == "C4":
        return [o for o in sm.oc_list() if not o & sm.OC_ST or o & sm.OC_RT]
    if name == "C1":
        return [0]
    return sm.oc_list()      # C2, C5, N2: all 30 OCs


def cpu_oracle_sample(name: str, budget_s: float = 12.0, acc=None, c=None):
    """Time the oracle (as it stands) on a bounded z-slab of the workload."""
    import oracle
    import stencil_inputs as si
    C, acc0, c0 = _config(name)
    if acc is None:
        acc, c = acc0, c0
    dims, steps, dtype = C["dims"], C["steps"], C["dtype"]
    r = (acc.shape[0] - 1) // 2
    threads = oracle.max_threads()
    if len(dims) == 2 and dims[0] * dims[1] <= 1 << 20:
        # small 2-D grid (C1): the whole workload, "CPU oracle in seconds" with 1
        # thread and with every thread (best of 5 each)
        u = si.make_field(dims, C["seed"], dtype)
        secs = {}
        for nt in (1, threads):
            best = math.inf
            for _ in range(5):
                t0 = time.perf_counter()
                oracle.sweep(u, acc, c, steps, dtype=dtype, nthreads=nt)
                best = min(best, time.perf_counter() - t0)
            secs[nt] = best
        dt = secs[threads]
        pts = (dims[0] - 2 * r) * (dims[1] - 2 * r) * steps
        return {"value": pts / dt / 1e9, "unit": "GStencil/s", "cores": threads, "kind": "oracle",
                "sample": (f"full {name} grid {dims}, {steps} steps: {secs[1]:.6f} s on 1 thread, "
                           f"{dt:.6f} s on {threads} threads (best of 5)"),
                "seconds": dt, "points": pts, "seconds_1_thread": round(secs[1], 6),
                "seconds_all_threads": round(dt, 6), "cpu_model": _cpu_model()}
    # probe with a thin slab (rows in 2-D, planes in 3-D), then size the sample to ~budget_s
    row = tuple(dims[1:])
    nz = 2 * r + 8
    u = si.make_field((nz,) + row, C["seed"], dtype, global_dims=dims)
    t0 = time.perf_counter()
    oracle.sweep(u, acc, c, 1, dtype=dtype)
    per_plane = (time.perf_counter() - t0) / (nz - 2 * r)
    full = dims[0] - 2 * r
    if per_plane * full * steps <= budget_s:          # the whole workload fits the budget
        planes, s_steps = full, steps
    else:
        s_steps = max(1, min(steps, int(budget_s / max(per_plane * full, 1e-9))))
        planes = int(max(8, min(full, budget_s / max(per_plane, 1e-9) / s_steps)))
    u = si.make_field((planes + 2 * r,) + row, C["seed"], dtype, global_dims=dims)
    t0 = time.perf_counter()
    oracle.sweep(u, acc, c, s_steps, dtype=dtype)
    dt = time.perf_counter() - t0
    inner = 1
    for d in row:
        inner *= d - 2 * r
    pts = planes * inner * s_steps
    unit = "planes" if len(dims) == 3 else "rows"
    return {"value": pts / dt / 1e9, "unit": "GStencil/s", "cores": threads, "kind": "oracle",
            "sample": (f"{planes}+{2 * r} {unit} x {'x'.join(map(str, row))} of the {name} grid, {s_steps} step(s), "
                       f"{dt:.2f} s; rate per interior update"), "seconds": dt, "points": pts}


def _cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def _cpu_workload(name: str, budget_s: float):
    """Oracle rate over every stencil of the workload: total sampled updates /
    total seconds (the same aggregation as the GPU value)."""
    items = _items(name)
    per = budget_s / len(items)
    samples = [cpu_oracle_sample(name, per, it["acc"], it["c"]) for it in items]
    pts = sum(x["points"] for x in samples)
    sec = sum(x["seconds"] for x in samples)
    # time-weighted: each stencil's full-workload time at its sampled rate
    C = _config(name)[0]
    tot_pts, tot_s = 0, 0.0
    for it, x in zip(items, samples):
        r = (it["acc"].shape[0] - 1) // 2
        n = 1
        for d in C["dims"]:
            n *= d - 2 * r
        tot_pts += n * C["steps"]
        tot_s += n * C["steps"] / (x["value"] * 1e9)
    v = tot_pts / tot_s / 1e9
    sample = "; ".join(f"{it['stencil']}: {x['sample']}" for it, x in zip(items, samples)) if len(items) > 1 \
        else samples[0]["sample"]
    out = {"value": v, "unit": "GStencil/s", "cores": samples[0]["cores"], "kind": "oracle", "sample": sample,
           "seconds": sec, "points": pts, "cpu_model": _cpu_model()}
    for k in ("seconds_1_thread", "seconds_all_threads"):
        if k in samples[0]:
            out[k] = samples[0][k]
    return out


def _workload_points(name: str) -> int:
    C = _config(name)[0]
    tot = 0
    for it in _items(name):
        r = (it["acc"].shape[0] - 1) // 2
        n = 1
        for d in C["dims"]:
            n *= d - 2 * r
        tot += n * C["steps"]
    return tot


def run_reference(args):
    rank, world, _ = _env_rank()
    if rank != 0:
        return 0
    name = args.config
    budget = max(2.0, min(60.0, 150.0 / max(1, args.steps + args.warmup)))
    vals = []
    cb = None
    for i in range(args.warmup + args.steps):
        cb = _cpu_workload(name, budget)
        if i >= args.warmup:
            vals.append(cb["value"])
    v = statistics.mean(vals)
    C = _config(name)[0]
    ms = _workload_points(name) / (v * 1e9) * 1e3
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": "GStencil/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": C["dtype"], "data": "synthetic",
        "config": {"workload": WORKLOADS.get(name, name), "grid": list(C["dims"]), "time_steps": C["steps"],
                   "stencils": [it["stencil"] for it in _items(name)],
                   "note": "oracle timed on a bounded slab sample; ms_per_step extrapolated to the full grid"},
        "cpu_baseline": {k: cb[k] for k in ("kind", "cores", "sample", "cpu_model", "seconds_1_thread",
                                            "seconds_all_threads") if k in cb} | {"value": v, "unit": "GStencil/s"},
        "e2e": {"value": v, "unit": "GStencil/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def kernel_key(config: str, lowered: str) -> str:
    """'C2:k_stream<16,8,1,8,0,0,1,1>' from a mangled NVRTC kernel name."""
    import re
    m = re.match(r"_ZN5smart(\d+)", lowered)
    if not m:
        return f"{config}:{lowered}"
    n = int(m.group(1))
    start = m.end()
    name = lowered[start:start + n]
    args = re.findall(r"L[ib](\d+)E", lowered[start + n:])
    return f"{config}:{name}<{','.join(args)}>"


def _pcie_probe(hin, hout, x, y):
    """Host-link context for e2e: one grid up, one grid down, and both at once
    (two streams), timed with CUDA events -- the bound the pipelined host path
     works against."""
    import torch
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    nb = x.numel() * x.element_size()

    def timed(fn):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        for s in (s1, s2):
            torch.cuda.current_stream().wait_stream(s)
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) * 1e-3

    def up():
        with torch.cuda.stream(s1):
            x.copy_(hin, non_blocking=True)

    def down():
        with torch.cuda.stream(s2):
            hout.copy_(y, non_blocking=True)

    for s in (s1, s2):
        s.wait_stream(torch.cuda.current_stream())
    t_up, t_down = timed(up), timed(down)
    t_both = timed(lambda: (up(), down()))
    return {"h2d": round(nb / t_up / 1e9, 1), "d2h": round(nb / t_down / 1e9, 1),
            "both_directions_total": round(2 * nb / t_both / 1e9, 1)}


def _traffic_from_profiles(key: str):
    """dram read+write bytes per launch from a committed `ncu --set full` capture."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    try:
        e = json.load(open(p)).get(key)
        return float(e["dram_bytes_per_launch"]) if e else None
    except Exception:
        return None


def measure_fma_peak(sm, dtype: str, local: int, seconds: float = 2.0) -> dict:
    """Measured FMA throughput of this GPU in `dtype` (stencil_fma_probe, a
    hand-written kernel of independent FMA chains on every SM): back-to-back
    launches of ~20 ms for `seconds`, SM clock sampled meanwhile. `sustained`
    (median of the second half, under the power cap) is the denominator of the
    "alu" roofline -- the FMA-bound stencil kernels are timed inside a long
    step; `burst` is the best launch."""
    import torch
    tdt = torch.float64 if dtype == "f64" else torch.float32
    sink = torch.zeros(1, dtype=tdt, device=f"cuda:{local}")
    stream = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    def once(iters):
        e0.record(stream)
        fl = sm.fma_probe(sink, iters, stream=stream)
        e1.record(stream)
        e1.synchronize()
        ms = e0.elapsed_time(e1)
        return fl / (ms * 1e-3) / 1e12, ms

    iters = 256
    once(iters)
    _, ms = once(iters)
    iters = max(1, int(iters * 20.0 / max(ms, 1e-3)))
    vals = []
    with ClockSampler(local) as clk:
        t_end = time.time() + seconds
        while time.time() < t_end or len(vals) < 6:
            vals.append(once(iters)[0])
    half = vals[len(vals) // 2:]
    c = clk.result()
    return {"sustained": round(statistics.median(half), 2), "burst": round(max(vals), 2), "unit": "TFLOP/s",
            "dtype": dtype, "launches": len(vals), "sm_mhz": c["sm_mhz"], "reasons": c["reasons"],
            "how": "stencil_fma_probe: 148 SMs x 8 CTAs x 256 threads, 12 independent FMA chains per thread with "
                   "immediate operands, ~20 ms launches back to back; 2 flops per FMA"}


def _roofline(name, sm, pinfo, oc, pts, steps, kern_ms, kern_n, total_ms, nsteps_timed, elem, dtype, peak, peak_kind,
              fma_peak=None):
    """Roofline of one stencil's sweep kernel: algorithmic bytes
    per launch (read + write every interior point once) / average launch time,
    and the FMA ceiling; the binding one is reported."""
    T = pinfo["params"]["tb_steps"] if oc & sm.OC_TB else 1
    groups = nsteps_timed * math.ceil(steps / T)
    bytes_per_launch = pts * 2 * elem
    flops_per_step = pts * 2 * pinfo["nnz"]    # one FMA per neighbour per point and step
    avg_launch_ms = kern_ms / max(groups, 1)
    achieved = bytes_per_launch / (avg_launch_ms * 1e-3) / 1e9
    # measured FMA peak (stencil_fma_probe, sustained); fallback: DESIGN.md §6's
    # derived 148 SM x 64 FMA/clk x 2 x 1.965 GHz = 37.2 TFLOP/s (FP32 x2)
    if fma_peak:
        fp_peak = fma_peak["sustained"]
        fp_kind = (f"measured (stencil_fma_probe, sustained, SM clock median {fma_peak['sm_mhz']} MHz; "
                   f"burst {fma_peak['burst']})")
    else:
        fp_peak = 148 * 64 * 2 * 1.965e9 / 1e12 * (1 if dtype == "f64" else 2)
        fp_kind = "derived (DESIGN.md §6)"
    achieved_fp = flops_per_step * nsteps_timed * steps / (kern_ms * 1e-3) / 1e12
    key = kernel_key(name, pinfo["kernel_name"])
    roof = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
            "frac": round(achieved / peak, 4), "traffic": _traffic_from_profiles(key),
            "peak_kind": peak_kind, "kernel": key,
            "launch_ms": round(avg_launch_ms, 4), "launches": kern_n,
            "kernel_share_of_step": round(kern_ms / max(total_ms, 1e-9), 4),
            "bytes_per_launch": bytes_per_launch, "time_steps_per_launch": T,
            "frac_of_spec_8tbs": round(achieved / HBM_SPEC_GBS, 4),
            "fp": {"achieved": round(achieved_fp, 2), "peak": round(fp_peak, 1), "unit": "TFLOP/s",
                   "frac": round(achieved_fp / fp_peak, 4), "peak_kind": fp_kind}}
    # FMA-bound stencils (C4, high-order random): the FP ceiling binds before HBM
    if flops_per_step / (fp_peak * 1e12) > bytes_per_launch / T / (peak * 1e9):
        roof.update({"bound": "alu", "achieved": round(achieved_fp, 2), "peak": round(fp_peak, 1),
                     "unit": "TFLOP/s", "frac": round(achieved_fp / fp_peak, 4),
                     "peak_kind": fp_kind,
                     "hbm": {"achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                             "frac": round(achieved / peak, 4)}})
        roof.pop("fp")
    return roof


def run_impl(args):
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_sunlyjlq22_b200 as sm

    rank, world, local = _env_rank()
    assert world == args.gpus, f"WORLD_SIZE={world} != --gpus {args.gpus}"
    assert torch.cuda.device_count() > local, f"rank {rank}: no GPU {local}"
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    sm.lib()
    name = args.config
    C = _config(name)[0]
    dims, steps, dtype = tuple(C["dims"]), C["steps"], C["dtype"]
    tdt = torch.float64 if dtype == "f64" else torch.float32
    elem = 8 if dtype == "f64" else 4
    peak, peak_kind = _peaks()
    items = _items(name)

    slab = (world > 1 or args.slab) and len(dims) == 3
    comm_owner = []

    def make_plan(acc, c, oc, params=None):
        """Plan on this rank's slab; the halo exchange (a7) runs on torch's NCCL
        communicator (N > 1) or on one library-owned communicator (N = 1)."""
        p = sm.Plan(dims, acc, c, dtype, oc, params)
        if slab:
            if world > 1:
                be = dist.distributed_c10d._get_default_group()._get_backend(dev)
                p.set_nccl_comm(be._comm_ptr(), rank, world)
            elif comm_owner:
                p.share_comm(comm_owner[0])
            else:
                p.set_comm(sm.nccl_unique_id(), rank, world)
                comm_owner.append(p)
        return p

    # every rank owns dims[0] planes of a global grid of depth world*dims[0]
    # (weak scaling); slab buffers carry G ghost planes on each side, G = the
    # stencil's own depth (4 x order), so in slab mode every stencil of a
    # multi-stencil workload (C5) gets its own input/output/workspace; otherwise
    # one pair (and one workspace) serves every stencil of the step.
    gdims = (dims[0] * world,) + dims[1:] if len(dims) == 3 else dims

    def alloc_bufs(it):
        probe = make_plan(it["acc"], it["c"], 0)
        G = probe.ghost
        xb = torch.zeros(probe.array_shape, dtype=tdt, device=dev)
        if len(dims) == 3:
            z0 = dims[0] * rank
            a, b = max(0, z0 - G), min(gdims[0], z0 + dims[0] + G)
            sm.fill_field(xb[a - (z0 - G):b - (z0 - G)], C["seed"], 0, origin=(a, 0, 0), global_dims=gdims)
        else:
            sm.fill_field(xb, C["seed"], 0)
        bufs = (xb, torch.empty_like(xb), torch.empty(probe.workspace_bytes() // elem, dtype=tdt, device=dev), G)
        del probe
        return bufs

    shared = None
    for it in items:
        if slab or shared is None:
            shared = alloc_bufs(it)
        it["x"], it["y"], it["ws"], it["G"] = shared
    x, y, ws, G = items[0]["x"], items[0]["y"], items[0]["ws"], max(it["G"] for it in items)
    stream = torch.cuda.current_stream()

    # ---- 1. label pass per stencil: every OC of the family, seeded settings (a8)
    ocs = _ocs_for(name, sm)
    p2p_flags, p2p_links = None, []
    if args.oc:
        ocs = [sm.oc_from_name(args.oc)]
    t_sw = time.time()
    for it in items:
        x, y, ws = it["x"], it["y"], it["ws"]
        base_plan = make_plan(it["acc"], it["c"], 0)
        base_plan.use_workspace(ws)
        info0 = base_plan.info
        it["points"] = info0["points"]          # this rank's interior points per time step
        it["nnz"] = info0["nnz"]
        if args.settings > 0 and len(ocs) > 1:
            sweep = base_plan.oc_sweep(x, y, steps=steps, settings_per_oc=args.settings, reps=3, seed=args.seed)
        else:
            sweep = {"oc_ids": sm.oc_list(), "times_ms": [math.inf] * sm.NUM_OC,
                     "best_params": [{}] * sm.NUM_OC, "best_oc": ocs[0]}
        per_oc, best_oc, best_t, best_p = {}, None, math.inf, None
        for oc, t, p in zip(sweep["oc_ids"], sweep["times_ms"], sweep["best_params"]):
            if oc not in ocs:
                continue
            gs = sm.gstencil_per_s(it["points"], steps, t) if math.isfinite(t) else None
            # a launch reads and writes the grid once (16 B / point in fp64) whatever
            # number of time steps it fuses: TB OCs move 2*elem/T bytes per update
            T_oc = (p or {}).get("tb_steps", 1) if oc & sm.OC_TB else 1
            per_oc[sm.oc_name(oc)] = {
                "ms": round(t, 4) if math.isfinite(t) else None,
                "gstencil_s": round(gs, 2) if gs else None,
                "time_steps_per_launch": T_oc,
                "hbm_frac_of_measured": round(gs * 2 * elem / T_oc / peak, 4) if gs else None,
                "hbm_frac_of_spec": round(gs * 2 * elem / T_oc / HBM_SPEC_GBS, 4) if gs else None,
                "infeasible": not math.isfinite(t),
            }
            if math.isfinite(t) and t < best_t:
                best_oc, best_t, best_p = oc, t, p
        # spatial tiling reported as its own entry (shared memory is a
        # Boolean parameter of base / BM / CM; the label pass draws it among the
        # sampled settings, so per_oc above may hold either form): the smem = 1
        # form of each, default tiles, median of 3 timed runs
        if args.tiling and args.settings > 0 and len(ocs) > 1:
            for oc in (0, sm.OC_BM, sm.OC_CM):
                if oc not in ocs:
                    continue
                key = sm.oc_name(oc) + "+tiling(smem=1)"
                try:
                    tp = make_plan(it["acc"], it["c"], oc, {"smem": 1})
                    tp.use_workspace(ws)
                    tp.run(x, y, steps)
                    ts = []
                    for _ in range(3):
                        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                        a.record(stream)
                        tp.run(x, y, steps)
                        b.record(stream)
                        b.synchronize()
                        ts.append(a.elapsed_time(b))
                    t = statistics.median(ts)
                    gs = sm.gstencil_per_s(it["points"], steps, t)
                    per_oc[key] = {"ms": round(t, 4), "gstencil_s": round(gs, 2), "time_steps_per_launch": 1,
                                   "hbm_frac_of_measured": round(gs * 2 * elem / peak, 4),
                                   "hbm_frac_of_spec": round(gs * 2 * elem / HBM_SPEC_GBS, 4), "infeasible": False,
                                   "kernel": tp.info["kernel_name"][:40]}
                    del tp
                except sm.StencilError as e:
                    per_oc[key] = {"ms": None, "gstencil_s": None, "infeasible": True, "why": str(e)[:120]}
        if best_oc is None:
            best_oc, best_p = ocs[0], None
        if args.params:
            best_p = json.loads(args.params)
        if world > 1:   # every rank must run the same OC: take rank 0's label
            obj = [best_oc, best_p]
            dist.broadcast_object_list(obj, src=0)
            best_oc, best_p = obj
        it["per_oc"], it["best_oc"] = per_oc, best_oc
        del base_plan
        if slab and args.transport == "p2p":
            # fused device-initiated halo: edge kernels store the neighbours'
            # ghost planes through peer memory (CUDA IPC), epochs in flag words
            from paper_conf_ipps_sunlyjlq22_b200 import p2p
            if p2p_flags is None:
                p2p_flags = p2p.new_flags(dev)
                if world == 1 and not dist.is_initialized():
                    dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % _free_port(), rank=0,
                                            world_size=1)
            it["plan"] = sm.Plan(dims, it["acc"], it["c"], dtype, best_oc, best_p or None)
            p2p_links.append(p2p.setup_p2p(it["plan"], x, y, ws, p2p_flags, rank, world))
        else:
            it["plan"] = make_plan(it["acc"], it["c"], best_oc, best_p or None)
            it["plan"].use_workspace(ws)
        it["pinfo"] = it["plan"].info
    sweep_s = time.time() - t_sw
    pts_rank = sum(it["points"] for it in items)
    pts_all = pts_rank
    if world > 1:
        t = torch.tensor([pts_rank], dtype=torch.float64, device=dev)
        dist.all_reduce(t)
        pts_all = int(t.item())

    # measured FMA peak (the "alu" roofline's denominator), before the timed region
    fma_peak = measure_fma_peak(sm, dtype, local)

    def step():
        for it in items:
            it["plan"].run(it["x"], it["y"], steps)

    # ---- 2. warm-up + timed steps (one step = every stencil of the workload)
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    launches0 = sm.launch_count()
    for it in items:
        it["plan"].kernel_time()                   # reset the per-launch accumulators
        it["plan"].set_timing(True)
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    # grids that fit the 126 MB L2 (C1: 0.5 MB) would be timed from L2: flush it
    # between the timed steps by writing a 256 MB buffer, outside the per-step
    # CUDA-event pairs (the time is their sum); larger grids stream through L2
    grid_bytes = max(it["x"].numel() for it in items) * elem
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev) if 2 * grid_bytes < L2_BYTES else None
    with ClockSampler(local) as clk:
        if flush is None:
            e0.record(stream)
            for _ in range(args.steps):
                step()
            e1.record(stream)
            torch.cuda.synchronize()
            total_ms = e0.elapsed_time(e1)
        else:
            evs = []
            for _ in range(args.steps):
                flush.fill_(1)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                step()
                b.record(stream)
                evs.append((a, b))
            torch.cuda.synchronize()
            total_ms = sum(a.elapsed_time(b) for a, b in evs)
    launches = sm.launch_count() - launches0
    l2_note = ("inputs (grid bytes) larger than the 126 MB L2; no flush needed" if flush is None else
               f"grid ({grid_bytes / 2**20:.1f} MiB) fits the 126 MB L2: a 256 MiB buffer is written between "
               "timed steps (not timed; per-step CUDA events summed)")
    for it in items:
        it["kern_ms"], it["kern_n"] = it["plan"].kernel_time()
        it["plan"].set_timing(False)
    if world > 1:
        t = torch.tensor([total_ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
        dist.barrier()
    ms_per_step = total_ms / args.steps
    value = pts_all * steps / (ms_per_step * 1e-3) / 1e9

    # ---- 3. roofline per stencil; the dominant kernel (largest share of the step) is reported
    for it in items:
        it["roofline"] = _roofline(name, sm, it["pinfo"], it["best_oc"], it["points"], steps, it["kern_ms"],
                                   it["kern_n"], total_ms, args.steps, elem, dtype, peak, peak_kind, fma_peak)
    dom = max(items, key=lambda it: it["kern_ms"])
    roofline = dict(dom["roofline"])
    if len(items) > 1:
        roofline["stencil"] = dom["stencil"]

    launch_bytes = sum(it["points"] * 2 * elem * math.ceil(steps / it["roofline"]["time_steps_per_launch"])
                       for it in items)
    hbm_gbs = launch_bytes / (ms_per_step * 1e-3) / 1e9

    # ---- 4. e2e through the public API with host buffers
    e2e = None
    if slab and args.transport == "p2p" and not args.no_e2e:
        # P2P slab plans run only on their registered buffers: the host path
        # (which stages into its own device buffers) does not apply
        e2e = {"value": None, "unsupported": "stencil_run_host does not run P2P-registered slab plans"}
    elif not args.no_e2e:
        # pinned host buffers of the largest stencil's array; each stencil runs
        # on a view of its own (slab) shape
        big = max(items, key=lambda it: it["x"].numel())["x"]
        hin = torch.empty(tuple(big.shape), dtype=tdt, pin_memory=True)
        hin.copy_(big.cpu())
        hout = torch.empty_like(hin).pin_memory()
        for it in items:
            n = it["x"].numel()
            it["hin"] = hin.view(-1)[:n].view(tuple(it["x"].shape))
            it["hout"] = hout.view(-1)[:n].view(tuple(it["x"].shape))
            it["plan"].run_host(it["hin"], it["hout"], steps)   # warm (allocates the plan's device buffers)
        n_e2e = max(1, min(3, args.steps))
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(n_e2e):
            for it in items:
                it["plan"].run_host(it["hin"], it["hout"], steps)
        torch.cuda.synchronize()
        e2e_ms = (time.perf_counter() - t0) * 1e3 / n_e2e
        if world > 1:
            t = torch.tensor([e2e_ms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e2e_ms = float(t.item())
        nbytes = sum(it["x"].numel() for it in items) * elem
        e2e = {"value": round(pts_all * steps / (e2e_ms * 1e-3) / 1e9, 3), "unit": "GStencil/s",
               "h2d_bytes_per_step": nbytes, "d2h_bytes_per_step": nbytes, "ms_per_step": round(e2e_ms, 3),
               "host_chunks": [it["plan"].info["host_chunks"] for it in items],
               "pcie_gbs": _pcie_probe(items[0]["hin"], items[0]["hout"], items[0]["x"], items[0]["y"])}
        for it in items:
            it.pop("hin", None), it.pop("hout", None)
        del hin, hout

    # ---- 5. CPU oracle beside it (rank 0, N = 1)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cb = _cpu_workload(name, args.cpu_budget)
        cpu = {k: cb[k] for k in ("value", "unit", "cores", "kind", "sample", "cpu_model", "seconds_1_thread",
                                  "seconds_all_threads") if k in cb}

    if rank == 0:
        first = items[0]
        line = {
            "metric": METRIC, "value": round(value, 2), "unit": "GStencil/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": dtype,
            "data": "synthetic",
            "config": {"workload": WORKLOADS.get(name, name), "grid_per_gpu": list(dims),
                       "global_grid": list(gdims), "time_steps_per_step": steps,
                       "stencil": first["stencil"] if len(items) == 1 else [it["stencil"] for it in items],
                       "oc": sm.oc_name(first["best_oc"]) if len(items) == 1
                       else {it["stencil"]: sm.oc_name(it["best_oc"]) for it in items},
                       "params": first["pinfo"]["params"] if len(items) == 1
                       else {it["stencil"]: it["pinfo"]["params"] for it in items},
                       "parallelism": (f"z-slabs x{world}, "
                                       + ("fused P2P halo (edge kernels store into peer ghost planes)"
                                          if args.transport == "p2p" else "NCCL halo exchange")
                                       + f" (ghost {G} planes), edge/interior overlap"
                                       if slab else "single GPU"),
                       "l2": l2_note},
            "roofline": roofline,
            # algorithmic bytes per step (every launch reads + writes its grid once;
            # TB launches fuse T steps) / step time, per GPU
            "hbm_frac_of_measured_per_gpu": round(hbm_gbs / peak, 4),
            "hbm_frac_of_spec_per_gpu": round(hbm_gbs / HBM_SPEC_GBS, 4),
            "fma_peak": fma_peak,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches,
            "clocks": clk.result(),
            "best_oc": sm.oc_name(first["best_oc"]) if len(items) == 1
            else {it["stencil"]: sm.oc_name(it["best_oc"]) for it in items},
            "per_oc": first["per_oc"] if len(items) == 1 else {it["stencil"]: it["per_oc"] for it in items},
            "label_sweep": {"settings_per_oc": args.settings, "reps": 3, "seconds": round(sweep_s, 1)},
        }
        if len(items) > 1:
            line["stencils"] = [{
                "stencil": it["stencil"], "order": (it["acc"].shape[0] - 1) // 2, "nnz": it["nnz"],
                "best_oc": sm.oc_name(it["best_oc"]),
                "gstencil_s": round(it["points"] * steps * args.steps / (it["kern_ms"] * 1e-3) / 1e9, 2)
                if it["kern_ms"] > 0 else None,
                "roofline": {k: it["roofline"][k] for k in ("bound", "achieved", "peak", "unit", "frac")}}
                for it in items]
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    # stdout carries exactly one JSON line: the image sets NCCL_DEBUG=VERSION,
    # whose banner NCCL prints to stdout at the first communicator (seen on the
    # --slab runs); WARN keeps warnings and drops the banner, and any other log
    # NCCL writes goes to stderr
    if os.environ.get("NCCL_DEBUG", "").upper() == "VERSION":
        os.environ["NCCL_DEBUG"] = "WARN"
    if os.environ.get("NCCL_DEBUG") and not os.environ.get("NCCL_DEBUG_FILE"):
        os.environ["NCCL_DEBUG_FILE"] = "/dev/stderr"
    ap = argparse.ArgumentParser(description=__doc__, formatter_class=argparse.RawDescriptionHelpFormatter)
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C5", choices=["C1", "C2", "C3", "C4", "C5", "N2"],
                    help="workload (default C5: the configuration BASELINE.json's metric is quoted on)")
    ap.add_argument("--settings", type=int, default=None,
                    help="settings per OC in the label pass (default 3; C5: 1, N2: 2)")
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--oc", default="", help="time this OC (skips the label pass); for profiling")
    ap.add_argument("--params", default="", help="JSON parameter setting for --oc")
    ap.add_argument("--cpu-budget", type=float, default=12.0)
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-tiling", dest="tiling", action="store_false",
                    help="skip the extra smem = 1 (spatial tiling) timings of base / BM / CM in per_oc")
    ap.add_argument("--slab", action="store_true", help="use the NCCL slab path even at N = 1")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "p2p"],
                    help="halo exchange of the timed slab runs: NCCL send/recv on a comm stream, or the fused "
                         "device-initiated P2P halo (edge kernels store into the neighbours' ghost planes)")
    args = ap.parse_args()
    if args.warmup < 3:
        ap.error("--warmup must be >= 3")
    if args.settings is None:
        args.settings = {"C5": 1, "N2": 2}.get(args.config, 3)
    if args.impl == "reference":
        return run_reference(args)
    world_env = os.environ.get("WORLD_SIZE")
    if world_env is None and args.gpus > 1:
        return spawn_ranks(args)
    if int(world_env or 1) != args.gpus:
        ap.error(f"--gpus {args.gpus} but WORLD_SIZE={world_env}: launch one rank per GPU")
    return run_impl(args)


def _rank_entry(local: int, args, port: int):
    os.environ.update(RANK=str(local), LOCAL_RANK=str(local), WORLD_SIZE=str(args.gpus),
                      MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    rc = run_impl(args)
    if rc:
        raise SystemExit(rc)


def spawn_ranks(args) -> int:
    """`--gpus N` without torchrun: spawn one process per GPU (NCCL over
    NVLink), each with RANK / LOCAL_RANK / WORLD_SIZE set as torchrun would;
    rank 0 prints the line. Fails loudly rather than timing fewer GPUs."""
    import torch
    import torch.multiprocessing as mp
    have = torch.cuda.device_count()
    if have < args.gpus:
        raise SystemExit(f"bench.py --gpus {args.gpus}: only {have} GPU(s) visible")
    mp.spawn(_rank_entry, args=(args, _free_port()), nprocs=args.gpus, join=True)
    return 0


if __name__ == "__main__":
    sys.exit(main())
