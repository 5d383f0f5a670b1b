"""Parity: stencil_oc_analysis (C ABI, host code in libstencilmart.so) vs the
OC-analysis oracle (oracle/oc_groups.py), SURVEY NEXT-4 (P:L89, P:L93,
P:L105-L107). No GPU needed.

* wins (integers from the times) bit-exact; gap (one division) bitwise;
* PCC within 1e-12 (the oracle sums exactly rounded, the product in its own
  order -- several fp64 results are correct);
* groups: where the oracle's |PCC| ranking has no rounding-level near-ties the
  grouping must equal the oracle's; always, it must be the single-linkage merge
  of the product's own PCC matrix (a valid result under rounding), and the
  representatives and class labels must follow from it exactly.
"""
import math

import numpy as np
import pytest

import paper_conf_ipps_sunlyjlq22_b200 as sm
from oracle import oc_groups as og

INF = math.inf


def _dataset_like(seed, n_st=64, n_oc=30, infeasible=0.05, dup=True):
    """Per-OC times shaped like a label sweep: stencil scale x OC effect, some
    OCs infeasible (+inf), some columns near-duplicates (OCs that only differ
    by a flag the stencil does not exercise)."""
    rng = np.random.default_rng(seed)
    t = np.exp(rng.uniform(-2, 3, size=(n_st, 1))) * np.exp(rng.normal(0, 0.5, size=(n_st, n_oc)))
    if dup:
        for a, b in ((1, 7), (2, 11), (20, 21)):
            if b < n_oc:
                t[:, b] = t[:, a] * (1.0 + 1e-3 * rng.normal(size=n_st))
    t[rng.uniform(size=t.shape) < infeasible] = INF
    return t


def _check(t, n_classes):
    got = sm.oc_analysis(t, n_classes)
    p_or = og.pcc(t)
    assert got["wins"].tolist() == og.wins(t).tolist()
    np.testing.assert_array_equal(got["gap"], og.gap(t))            # NaN == NaN here
    np.testing.assert_allclose(got["pcc"], p_or, rtol=0, atol=1e-12)
    # a valid single-linkage result on the product's PCC, with the representatives
    # and labels that grouping implies
    gid_p, reps_p = og.groups_from_pcc(t, np.asarray(got["pcc"]), n_classes)
    assert got["group"] == gid_p
    assert got["representative"] == reps_p
    assert got["labels"] == og.class_labels(t, gid_p)
    if og.ranking_is_tie_free(p_or):                                  # unambiguous: the oracle's grouping
        gid, reps = og.groups(t, n_classes)
        assert got["group"] == gid and got["representative"] == reps
    return og.ranking_is_tie_free(p_or)


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("n_classes", [5, 1, 12])
def test_parity_dataset_like(seed, n_classes):
    assert _check(_dataset_like(seed), n_classes)    # these rankings have no near-ties


def test_parity_edge_cases():
    rng = np.random.default_rng(7)
    t = _dataset_like(8, n_st=10, n_oc=6, dup=False)
    t[3, :] = INF                                   # a stencil nothing ran on
    t[:, 4] = INF                                   # an OC that never ran (PCC 0 with all)
    _check(t, 5)
    _check(t[:2], 5)                                # < 3 stencils: every PCC 0
    _check(np.ones((5, 4)), 2)                      # constant perf: zero variance, all ties
    _check(_dataset_like(9, n_oc=3), 5)             # fewer OCs than classes
    _check(np.round(rng.uniform(1, 3, size=(20, 8)), 1), 3)   # many exact time ties


def test_empty_dataset():
    got = sm.oc_analysis(np.zeros((0, 30)), 5)
    assert got["labels"] == [] and got["wins"].tolist() == [0] * 30
    assert got["group"] == og.groups(np.zeros((0, 30)), 5)[0]


def test_invalid_arguments():
    with pytest.raises(sm.StencilError):
        sm.oc_analysis(np.ones((3, 4)), 0)
    with pytest.raises(sm.StencilError):
        sm.oc_analysis(np.ones((3, 65)), 5)
