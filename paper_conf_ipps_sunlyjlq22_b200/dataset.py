"""Stencil dataset rows: the label generator's full output.

"the performance of each stencil input is profiled with different OCs on the
target GPU, and the OC with the best performance is labeled ... Each parameter
setting and its corresponding execution time are also stored in the stencil
dataset" (§IV-A). One JSON line per (stencil, OC, setting) plus one
label line per stencil; features come from the Table II extractor and the 9^d
tensor of Fig. 6 (both in libstencilmart.so). Files are append-only JSONL, so an
interrupted run resumes by skipping stencil ids already labelled (`resume`
first cuts a torn tail: a partial last line and the setting rows of a stencil
whose label line was never written).
"""
from __future__ import annotations

import json
import math
import os
from typing import Iterable, List, Optional, Sequence, Set

import numpy as np

from .binding import Plan, embed_tensor, features, fill_field, oc_name


def done_ids(path: str) -> Set[str]:
    out: Set[str] = set()
    if os.path.exists(path):
        with open(path) as f:
            for line in f:
                try:
                    d = json.loads(line)
                except json.JSONDecodeError:
                    continue                      # a torn last line of an interrupted run
                if d.get("kind") == "label":
                    out.add(d["stencil_id"])
    return out


def resume(path: str) -> Set[str]:
    """Make an interrupted dataset file appendable and return the labelled ids.

    A stencil's rows are appended as one block ending with its label line, so
    everything after the last complete label line -- a torn last line, or the
    setting rows of a stencil whose label never landed -- belongs to a stencil
    that must be swept again: the file is truncated there (it would otherwise
    leave duplicate setting rows, or glue the next row onto the torn line)."""
    if not os.path.exists(path):
        return set()
    keep = 0
    out: Set[str] = set()
    with open(path, "rb") as f:
        pos = 0
        for raw in f:
            pos += len(raw)
            if not raw.endswith(b"\n"):
                break                             # torn last line
            try:
                d = json.loads(raw)
            except json.JSONDecodeError:
                break
            if d.get("kind") == "label":
                out.add(d["stencil_id"])
                keep = pos
    if keep != os.path.getsize(path):
        with open(path, "r+b") as f:
            f.truncate(keep)
    return out


def label_stencil(stencil_id: str, access: np.ndarray, coeffs: np.ndarray, dims: Sequence[int], dtype: str,
                  steps: int = 4, settings_per_oc: int = 4, reps: int = 3, seed: int = 0,
                  field_seed: int = 1) -> List[dict]:
    """Sweep one stencil under all 30 OCs on the current GPU; return its rows."""
    import torch
    tdt = torch.float64 if dtype == "f64" else torch.float32
    plan = Plan(dims, access, coeffs, dtype, 0)
    x = torch.empty(plan.array_shape, dtype=tdt, device="cuda")
    fill_field(x, field_seed)
    y = torch.empty_like(x)
    res = plan.oc_sweep(x, y, steps, settings_per_oc=settings_per_oc, reps=reps, seed=seed)
    feats = features(access)
    tensor = "".join(str(int(v)) for v in embed_tensor(access).ravel())
    common = {"stencil_id": stencil_id, "ndim": int(access.ndim), "dims": list(dims), "dtype": dtype,
              "steps": steps}
    rows = []
    for r in res["rows"]:
        t = r["time_ms"]
        rows.append(dict(common, kind="setting", oc=r["oc"], oc_name=r["oc_name"], setting=r["setting"],
                         params=r["params"], time_ms=t if math.isfinite(t) else None, status=r["status"]))
    rows.append(dict(common, kind="label", best_oc=res["best_oc"], best_oc_name=oc_name(res["best_oc"]),
                     oc_times_ms={oc_name(o): (t if math.isfinite(t) else None)
                                  for o, t in zip(res["oc_ids"], res["times_ms"])},
                     features=feats, tensor9=tensor))
    return rows


def append_rows(path: str, rows: Iterable[dict]) -> None:
    with open(path, "a") as f:
        for r in rows:
            f.write(json.dumps(r) + "\n")
        f.flush()
        os.fsync(f.fileno())


def load_matrix(path: str, ndim: Optional[int] = None):
    """(stencil ids, OC names, [n_stencils][30] per-OC shortest times in ms, +inf =
    infeasible) from the label lines of a dataset file -- the input of the OC
    analysis ("the shortest execution time of each OC under different
    parameter settings is used for OC selection")."""
    from .binding import oc_list
    names = [oc_name(o) for o in oc_list()]
    ids, rows = [], []
    with open(path) as f:
        for line in f:
            try:
                d = json.loads(line)
            except json.JSONDecodeError:
                continue
            if d.get("kind") != "label" or (ndim is not None and d.get("ndim") != ndim):
                continue
            t = d["oc_times_ms"]
            ids.append(d["stencil_id"])
            rows.append([math.inf if t.get(n) is None else float(t[n]) for n in names])
    return ids, names, np.array(rows, dtype=np.float64).reshape(len(rows), len(names))
