"""OC analysis oracle -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Plain numpy / pure-Python statement of the analysis the paper runs between
labelling and classification, on a (stencil x OC) matrix of per-OC shortest
times (the label generator's output, §IV-A, §V-A.2). Never
imported by the product package. Citations are PAPER.md line numbers.

* :func:`gap`      -- Fig. 1 (§III-A): best OC's performance normalised to
                      the worst OC's, per stencil, infeasible OCs left out
                      ("cases where OC crashes ... not reflected").
* :func:`wins`     -- Fig. 2 (§III-B): number of stencils each OC is the
                      best for (best = shortest time, ties -> smallest id,
                      reading C-11).
* :func:`pcc`      -- Fig. 3 (§III-C): Pearson correlation
                      coefficient between the performance of two OCs over the
                      stencils. Readings (DESIGN.md R-PCC): "performance" of OC o
                      on stencil s is t_best(s) / t(s, o) (normalised per
                      stencil, so the stencil's own scale does not dominate);
                      a pair uses the stencils where both OCs are feasible
                      (pairwise-complete); a pair with < 3 common stencils or
                      zero variance has PCC 0.
* :func:`groups`   -- the merge of P:L107 / P:L186 / P:L234: pairs ordered by
                      |PCC| (descending; ties -> (a, b) ascending) are merged
                      one by one (union of their groups) until n_classes groups
                      remain; from each group "the OC that obtains the best
                      performance under more cases (Figure 2)" is the
                      prediction target (ties -> smallest id). Groups are
                      numbered by their smallest member id.
* :func:`class_labels` -- the class of each stencil = group of its best OC.

Pinned by tests/test_oc_groups_pins.py against scipy (pearsonr, single-linkage
hierarchical clustering on 1 - |PCC|), brute force and hand-built cases.
"""
from __future__ import annotations

import math
from typing import Dict, List, Sequence, Tuple

import numpy as np


def _finite(t: float) -> bool:
    return t is not None and math.isfinite(t) and t > 0


def best_index(row: Sequence[float]) -> int:
    """Column of the shortest finite time; ties -> smallest column; -1 if none."""
    best, bt = -1, math.inf
    for j, t in enumerate(row):
        if _finite(t) and t < bt:
            best, bt = j, t
    return best


def gap(times: np.ndarray) -> np.ndarray:
    """Per stencil: worst finite time / best finite time (Fig. 1); NaN if no OC ran."""
    out = np.full(times.shape[0], np.nan)
    for i in range(times.shape[0]):
        f = [t for t in times[i] if _finite(t)]
        if f:
            out[i] = max(f) / min(f)
    return out


def wins(times: np.ndarray) -> np.ndarray:
    """Fig. 2: for each OC column, the number of stencils it is the best for."""
    w = np.zeros(times.shape[1], dtype=np.int64)
    for i in range(times.shape[0]):
        b = best_index(times[i])
        if b >= 0:
            w[b] += 1
    return w


def performance(times: np.ndarray) -> np.ndarray:
    """perf[s, o] = t_best(s) / t(s, o); NaN where OC o did not run on s."""
    perf = np.full(times.shape, np.nan)
    for i in range(times.shape[0]):
        b = best_index(times[i])
        if b < 0:
            continue
        for j in range(times.shape[1]):
            if _finite(times[i, j]):
                perf[i, j] = times[i, b] / times[i, j]
    return perf


def pearson(x: Sequence[float], y: Sequence[float]) -> float:
    """Textbook PCC: cov(x, y) / (sd(x) sd(y)); 0 if undefined (< 3 points or zero variance).

    Sums are exactly rounded (math.fsum): the oracle states the definition, it
    does not mimic any summation order of the product (tests compare the PCC at
    a tolerance and the groups only where the ranking is not a rounding tie)."""
    n = len(x)
    if n < 3:
        return 0.0
    mx = math.fsum(x) / n
    my = math.fsum(y) / n
    sxy = math.fsum((a - mx) * (b - my) for a, b in zip(x, y))
    sxx = math.fsum((a - mx) * (a - mx) for a in x)
    syy = math.fsum((b - my) * (b - my) for b in y)
    if sxx == 0.0 or syy == 0.0:
        return 0.0
    return sxy / math.sqrt(sxx * syy)


def pcc(times: np.ndarray) -> np.ndarray:
    """[n_oc, n_oc] PCC matrix of per-stencil normalised performance (diagonal 1)."""
    perf = performance(times)
    k = times.shape[1]
    m = np.eye(k)
    for a in range(k):
        for b in range(a + 1, k):
            xs, ys = [], []
            for i in range(times.shape[0]):
                if not (math.isnan(perf[i, a]) or math.isnan(perf[i, b])):
                    xs.append(float(perf[i, a]))
                    ys.append(float(perf[i, b]))
            m[a, b] = m[b, a] = pearson(xs, ys)
    return m


def ranked_pairs(p: np.ndarray) -> List[Tuple[float, int, int]]:
    """Pairs (|PCC|, a, b), a < b, by |PCC| descending, ties -> (a, b) ascending."""
    k = p.shape[0]
    pairs = [(abs(float(p[a, b])), a, b) for a in range(k) for b in range(a + 1, k)]
    pairs.sort(key=lambda t: (-t[0], t[1], t[2]))
    return pairs


def groups(times: np.ndarray, n_classes: int = 5) -> Tuple[List[int], List[int]]:
    """(group id per OC column, representative column per group).

    Merge pairs in ranked order until n_classes groups remain ("the OC
    pairs ... can be grouped to reduce the classes to be predicted"; P:L234:
    "reduce the number of predicted OCs to 5").
    """
    return groups_from_pcc(times, pcc(times), n_classes)


def ranking_is_tie_free(p: np.ndarray, tol: float = 1e-9) -> bool:
    """True when no two pairs' |PCC| differ by a rounding-level amount (0 < d <= tol):
    then any PCC within tol/2 of these values ranks the pairs the same way."""
    v = sorted(r[0] for r in ranked_pairs(p))
    return all(not (0.0 < b - a <= tol) for a, b in zip(v, v[1:]))


def groups_from_pcc(times: np.ndarray, p: np.ndarray, n_classes: int = 5) -> Tuple[List[int], List[int]]:
    """The merge of :func:`groups` on a given PCC matrix `p`."""
    k = times.shape[1]
    member = [{j} for j in range(k)]          # plain sets, merged explicitly
    where = list(range(k))
    count = k
    for _, a, b in ranked_pairs(p):
        if count <= n_classes:
            break
        ga, gb = where[a], where[b]
        if ga == gb:
            continue
        member[ga] |= member[gb]
        for j in member[gb]:
            where[j] = ga
        member[gb] = set()
        count -= 1
    roots = sorted({min(member[g]) for g in set(where)})
    gid = [roots.index(min(member[where[j]])) for j in range(k)]
    w = wins(times)
    reps = []
    for c in range(len(roots)):
        cols = [j for j in range(k) if gid[j] == c]
        reps.append(max(cols, key=lambda j: (w[j], -j)))
    return gid, reps


def class_labels(times: np.ndarray, gid: Sequence[int]) -> List[int]:
    """Class of each stencil = group of its best OC (-1 if no OC ran)."""
    out = []
    for i in range(times.shape[0]):
        b = best_index(times[i])
        out.append(gid[b] if b >= 0 else -1)
    return out


def top_pcc(p: np.ndarray, n: int = 100) -> List[Tuple[float, int, int]]:
    """Fig. 3: the top-n pairs by |PCC|."""
    return ranked_pairs(p)[:n]


def summary(times: np.ndarray, n_classes: int = 5) -> Dict[str, object]:
    g = gap(times)
    gid, reps = groups(times, n_classes)
    return {"mean_gap": float(np.nanmean(g)) if np.any(~np.isnan(g)) else None,
            "wins": wins(times).tolist(), "group": gid, "representative": reps,
            "classes": class_labels(times, gid)}
