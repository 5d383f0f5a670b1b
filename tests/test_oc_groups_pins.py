"""Pins of the OC-analysis oracle (PAPER.md P:L89, P:L93, P:L105-L107,
P:L186) against library routines and hand-built cases (no GPU).

Expected values come from scipy (pearsonr; single-linkage hierarchical
clustering, whose merge order on the distance 1 - |PCC| is exactly "merge the
most correlated pair next"), closed forms and hand-built matrices -- never from
the oracle itself.
"""
import math

import numpy as np
import pytest
from scipy.cluster.hierarchy import fcluster, linkage
from scipy.spatial.distance import squareform
from scipy.stats import pearsonr

from oracle import oc_groups as og

INF = math.inf


def _partition(labels):
    out = {}
    for j, g in enumerate(labels):
        out.setdefault(g, set()).add(j)
    return sorted(frozenset(s) for s in out.values())


def _random_times(rng, n_st=40, n_oc=12, infeasible=0.0):
    scale = np.exp(rng.uniform(-3, 3, size=(n_st, 1)))           # stencils differ in size
    eff = np.exp(rng.normal(0, 0.6, size=(n_st, n_oc)))          # OC effect per stencil
    t = scale * eff
    if infeasible:
        t[rng.uniform(size=t.shape) < infeasible] = INF
    return t


def test_pearson_matches_scipy():
    rng = np.random.default_rng(1)
    for n in (3, 7, 50):
        x, y = rng.normal(size=n), rng.normal(size=n) + 0.3 * np.arange(n)
        assert og.pearson(list(x), list(y)) == pytest.approx(pearsonr(x, y)[0], abs=1e-12)


def test_pearson_degenerate_cases():
    assert og.pearson([1.0, 2.0], [3.0, 4.0]) == 0.0            # < 3 points
    assert og.pearson([1.0, 1.0, 1.0], [1.0, 2.0, 3.0]) == 0.0  # zero variance
    assert og.pearson([1.0, 2.0, 3.0], [2.0, 4.0, 6.0]) == pytest.approx(1.0)
    assert og.pearson([1.0, 2.0, 3.0], [3.0, 2.0, 1.0]) == pytest.approx(-1.0)


def test_pcc_matrix_matches_corrcoef_when_all_feasible():
    rng = np.random.default_rng(2)
    t = _random_times(rng)
    perf = t.min(axis=1, keepdims=True) / t                      # t_best / t  (reading R-PCC)
    ref = np.corrcoef(perf, rowvar=False)
    np.testing.assert_allclose(og.pcc(t), ref, atol=1e-12)


def test_pcc_pairwise_complete_with_infeasible():
    rng = np.random.default_rng(3)
    t = _random_times(rng, infeasible=0.15)
    p = og.pcc(t)
    perf = og.performance(t)
    for a, b in ((0, 1), (3, 7), (5, 11)):
        ok = ~np.isnan(perf[:, a]) & ~np.isnan(perf[:, b])
        assert p[a, b] == pytest.approx(pearsonr(perf[ok, a], perf[ok, b])[0], abs=1e-12)


def test_pcc_invariant_to_stencil_scale():
    rng = np.random.default_rng(4)
    t = _random_times(rng)
    s = np.exp(rng.uniform(-2, 2, size=(t.shape[0], 1)))
    np.testing.assert_allclose(og.pcc(t), og.pcc(t * s), atol=1e-12)


@pytest.mark.parametrize("seed,n_classes", [(5, 5), (6, 3), (7, 8), (8, 1)])
def test_groups_equal_single_linkage(seed, n_classes):
    """Merging pairs by descending |PCC| = single linkage on 1 - |PCC| (scipy)."""
    rng = np.random.default_rng(seed)
    t = _random_times(rng)
    p = og.pcc(t)
    d = 1.0 - np.abs(p)
    np.fill_diagonal(d, 0.0)
    z = linkage(squareform(d, checks=False), method="single")
    assert len(set(np.round(z[:, 2], 14))) == len(z)              # no tied merge heights
    ref = fcluster(z, n_classes, criterion="maxclust")
    gid, reps = og.groups(t, n_classes)
    assert len(set(gid)) == n_classes
    assert _partition(gid) == _partition(ref)


def test_groups_duplicates_merge_first():
    """OC pairs with identical (scaled) behaviour have PCC 1 and merge first."""
    rng = np.random.default_rng(9)
    base = _random_times(rng, n_oc=3)
    t = np.concatenate([base, base * 1.5], axis=1)               # OC j+3 = 1.5 x OC j
    gid, _ = og.groups(t, 3)
    assert _partition(gid) == sorted([frozenset({0, 3}), frozenset({1, 4}), frozenset({2, 5})])
    assert gid == [0, 1, 2, 0, 1, 2]                              # numbered by smallest member


def test_gap_wins_and_labels_hand_built():
    t = np.array([[1.0, 2.0, INF, 4.0],
                  [3.0, 3.0, 1.5, 6.0],      # best = column 2
                  [2.0, 2.0, 5.0, 8.0],      # tie 0/1 -> 0
                  [INF, INF, INF, INF]])     # nothing ran
    g = og.gap(t)
    assert g[0] == 4.0 and g[1] == 4.0 and g[2] == 4.0 and math.isnan(g[3])
    assert og.wins(t).tolist() == [2, 0, 1, 0]
    gid = [0, 0, 1, 1]
    assert og.class_labels(t, gid) == [0, 1, 0, -1]


def test_representative_is_group_member_with_most_wins():
    rng = np.random.default_rng(10)
    t = _random_times(rng, n_st=60, n_oc=10)
    gid, reps = og.groups(t, 4)
    w = og.wins(t)
    for c, rep in enumerate(reps):
        members = [j for j in range(t.shape[1]) if gid[j] == c]
        assert gid[rep] == c
        assert w[rep] == max(w[j] for j in members)
        assert rep == min(j for j in members if w[j] == w[rep])


def test_groups_all_when_n_classes_ge_ocs():
    rng = np.random.default_rng(11)
    t = _random_times(rng, n_oc=5)
    gid, reps = og.groups(t, 5)
    assert gid == [0, 1, 2, 3, 4] and reps == [0, 1, 2, 3, 4]
