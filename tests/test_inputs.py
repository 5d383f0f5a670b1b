"""Input generators: counter-based field (C-3) and Algorithm 1.

Algorithm 1 is random, so it is pinned by invariants G1-G4.
"""
import itertools
import math

import numpy as np
import pytest

import stencil_inputs as si


def _splitmix_scalar(seed, g):
    """Independent pure-Python-int statement of h(seed, g) (C-3)."""
    M = (1 << 64) - 1
    key = (seed * 0xD1B54A32D192ED03) & M
    z = ((g ^ key) + 0x9E3779B97F4A7C15) & M
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M
    return z ^ (z >> 31)


def test_hash_matches_scalar_statement():
    g = np.array([0, 1, 2, 12345678901, (1 << 40) + 7], dtype=np.uint64)
    got = si.hash_index(77, g)
    for gi, hi in zip(g.tolist(), got.tolist()):
        assert hi == _splitmix_scalar(77, gi)


def test_field_ranges_and_subbox():
    f = si.make_field((9, 10, 11), 5, "f64")
    assert f.dtype == np.float64 and f.min() >= 1.0 and f.max() < 2.0
    f32 = si.make_field((9, 10, 11), 5, "f32")
    assert f32.dtype == np.float32 and f32.min() >= 1.0 and f32.max() < 2.0
    sub = si.make_field((3, 4, 5), 5, "f64", origin=(2, 3, 4), global_dims=(9, 10, 11))
    assert np.array_equal(sub, f[2:5, 3:7, 4:9])
    i = si.make_field((50, 60), 1, "f64", kind="int1023")
    assert np.all(i == np.round(i)) and i.min() >= -1023 and i.max() <= 1023


def test_config_stencils_sum_to_one():
    for name in ("heat2d", "heat3d", "star25", "box125", "random3d:3:2"):
        acc, c = si.config_stencil(name)
        assert abs(c.sum() - 1.0) < 1e-15
        assert np.all(c[acc == 0] == 0.0)
        r = (acc.shape[0] - 1) // 2
        assert acc[(r,) * acc.ndim] == 1
    assert si.heat3d()[0].sum() == 7 and si.star25()[0].sum() == 25 and si.box125()[0].sum() == 125


@pytest.mark.parametrize("ndim", [2, 3])
@pytest.mark.parametrize("order", [1, 2, 3, 4])
def test_algorithm1_invariants(ndim, order):
    for seed in range(4):
        acc, np_list = si.random_stencil(ndim, order, seed)
        r = order
        # G1: centre accessed
        assert acc[(r,) * ndim] == 1
        # G3: max ring = N exactly (order = max extent)
        offs = [tuple(o) for o in (np.argwhere(acc) - r)]
        assert max(si.ring_index(o) for o in offs) == order
        # npList[k] lies in ring k (plus, at k = 2, possibly the centre)
        for k, s in enumerate(np_list, start=1):
            assert all(si.ring_index(q) == k or (k == 2 and si.ring_index(q) == 0) for q in s)
            assert any(si.ring_index(q) == k for q in s)
        # G2: every selected ring-k point (k >= 2) has a Moore neighbour selected at k-1
        for k in range(2, order + 1):
            prev = np_list[k - 2]
            for q in np_list[k - 1]:
                if si.ring_index(q) != k:
                    continue
                assert any(max(abs(a - b) for a, b in zip(q, p)) == 1 for p in prev)


@pytest.mark.parametrize("ndim", [2, 3])
def test_algorithm1_full_box_and_determinism(ndim):
    for order in (1, 2, 3, 4):
        acc, _ = si.random_stencil(ndim, order, 3, p=1.0)      # G4
        assert acc.sum() == (2 * order + 1) ** ndim
    a1, _ = si.random_stencil(ndim, 3, 123)
    a2, _ = si.random_stencil(ndim, 3, 123)
    assert np.array_equal(a1, a2)


def _moore_ring(points, ndim, k):
    """Independent Moore-neighbourhood expansion (itertools), restricted to ring k."""
    out = set()
    for q in points:
        for d in itertools.product((-1, 0, 1), repeat=ndim):
            if any(d):
                c = tuple(a + b for a, b in zip(q, d))
                if max(abs(v) for v in c) == k:
                    out.add(c)
    return out


def _trunc_binom(n, p):
    """Mean and variance of Binomial(n, p) conditioned on >= 1 success (the
    redraw of reading C-7)."""
    z = 1.0 - (1.0 - p) ** n
    m1 = n * p / z
    m2 = (n * p * (1.0 - p) + (n * p) ** 2) / z
    return m1, m2 - m1 * m1


@pytest.mark.parametrize("ndim,samples", [(2, 3000), (3, 1500)])
def test_algorithm1_order1_distribution(ndim, samples):
    """G5 (Alg. 1 lines 4-6; reading C-7): at order 1 every one of
    the 3^d - 1 Moore neighbours of the centre is a candidate and is kept with
    probability p / (1 - (1-p)^M); the ring-1 count is a truncated binomial.
    A star-only neighbourhood or a biased draw fails here."""
    M = 3 ** ndim - 1
    p = 0.5
    pk = p / (1.0 - (1.0 - p) ** M)
    freq = {}
    counts = []
    for s in range(samples):
        _, np_list = si.random_stencil(ndim, 1, 10_000 + s)
        counts.append(len(np_list[0]))
        for q in np_list[0]:
            freq[q] = freq.get(q, 0) + 1
    assert set(freq) == _moore_ring([(0,) * ndim], ndim, 1)
    sd = math.sqrt(pk * (1 - pk) / samples)
    for q, f in freq.items():
        assert abs(f / samples - pk) < 5 * sd, (q, f / samples, pk)
    m, v = _trunc_binom(M, p)
    assert abs(np.mean(counts) - m) < 5 * math.sqrt(v / samples)


@pytest.mark.parametrize("ndim,order,samples", [(2, 2, 1500), (3, 2, 600), (2, 3, 800), (3, 3, 300)])
def test_algorithm1_higher_order_conditional_counts(ndim, order, samples):
    """G6 (Alg. 1 lines 8-14): given the order-(k-1) selection S,
    the ring-k candidates are exactly the Moore neighbours of S lying on ring k
    (rings k-1 and k-2 deleted), each kept with probability p under the redraw
    of reading C-7. Summed over samples, (count - E[count | S]) is centred with
    the truncated-binomial variance: candidates drawn from only part of S (e.g.
    the previous ring's axis points) or a different keep probability shift the
    mean by many sigmas. Ring deletion itself is pinned by G2/G3 above."""
    p = 0.5
    dev, var = 0.0, 0.0
    for s in range(samples):
        _, np_list = si.random_stencil(ndim, order, 20_000 + s)
        prev = np_list[order - 2]
        cand = _moore_ring(prev, ndim, order)
        got = [q for q in np_list[order - 1] if si.ring_index(q) == order]
        assert set(got) <= cand
        m, v = _trunc_binom(len(cand), p)
        dev += len(got) - m
        var += v
    assert abs(dev) < 5 * math.sqrt(var)
