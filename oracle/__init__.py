"""oracle/ -- TEST INFRASTRUCTURE ONLY (PAPER.md StencilMART, IPDPS'22).

A plain, slow, obviously correct CPU statement of what the hot path computes.
Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import, call, link or execute anything here. The
product path (``paper_conf_ipps_sunlyjlq22_b200``) never imports it and the
oracle never imports the product; both may use ``stencil_inputs`` (seeded input
generators, no stencil arithmetic).

Functions and the passages they follow:

* :func:`sweep` -- the stencil update (§I, §IV-B) with the frame
  rule C-1, fp64 plain loops in C (``stencil_oracle.c``).
  Pinned by tests/test_oracle_pins.py: library conv3d/conv2d (P1), constant
  field (P2), linear field (P3), heat eigenmode (P4), Fourier symbol (P5), time
  composition (P6), dyadic-exact bitwise (P7), per-point brute force over the
  dense tensor (P8), linearity/translation (P11).
* :func:`sweep_points` -- the same definition evaluated at sampled points of an
  arbitrarily large grid via the dependency cone (radius steps*r), the input
  regenerated from the counter-based generator. Pinned against :func:`sweep`.
* :func:`valid_ocs` -- Table I constraints. Pinned by the
  closed-form count 6 + 24 = 30 and explicit membership checks.
* :func:`best_oc` -- label = OC with the shortest time,
  infeasible (+inf) never best, ties -> smallest id (reading C-11). Pinned by
  hand-built vectors.
* :func:`features` -- Table II features. Pinned by star / box
  closed forms (nnz = 2dr+1, (2r+1)^d; ring sizes (2k+1)^d - (2k-1)^d).
* :mod:`oracle.oc_groups` -- the OC analysis between labelling and
  classification: Fig. 1 gap, Fig. 2 wins,
  Fig. 3 pairwise PCC and the PCC merge into 5 classes (P:L107,
  P:L186). Pinned by tests/test_oc_groups_pins.py (scipy pearsonr,
  scipy single-linkage clustering, hand-built matrices).
"""
from . import oc_groups
from .oracle import (OC_BITS, best_oc, build_oracle, features, max_threads, oc_name,
                     sweep, sweep_points, valid_ocs)

__all__ = ["oc_groups", "OC_BITS", "best_oc", "build_oracle", "features", "max_threads", "oc_name",
           "sweep", "sweep_points", "valid_ocs"]
