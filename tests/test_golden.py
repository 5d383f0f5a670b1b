"""Golden fixtures transcribed from the paper (tests/golden/, each line cited in
the file itself), checked against the oracle and the C-ABI's host logic (no GPU).

The OC lattice is re-derived here from the transcribed Table I rows by brute
force over all 2^6 subsets of the six optimizations -- a different route from
oracle.valid_ocs(), which hard-codes the two exclusion rules.
"""
import itertools
import pathlib

import oracle

GOLDEN = pathlib.Path(__file__).parent / "golden"


def _table1():
    rows, extra = [], {}
    for line in (GOLDEN / "table1_oc_constraints.txt").read_text().splitlines():
        line = line.split("#", 1)[0].strip()
        if not line:
            continue
        f = line.split()
        if f[0].isdigit():
            rows.append((int(f[0]), f[1], f[2], f[3]))
        else:
            extra[f[0]] = f[1:]
    return rows, extra


def _lattice_from_table1(rows):
    abbrevs = [r[2] for r in rows]
    valid = []
    for bits in itertools.product([False, True], repeat=len(abbrevs)):
        on = {a for a, b in zip(abbrevs, bits) if b}
        ok = True
        for _, _, a, c in rows:
            if a not in on or c == "-":
                continue
            kind, other = c.split(":")
            if kind == "excl" and other in on:
                ok = False
            if kind == "requires" and other not in on:
                ok = False
        if ok:
            valid.append(frozenset(on))
    return valid


def _mask(on):
    m = 0
    for a in on:
        m |= oracle.OC_BITS[a]
    return m


def test_table1_rows_transcribed():
    rows, _ = _table1()
    assert [r[0] for r in rows] == [1, 2, 3, 4, 5, 6]
    assert [r[2] for r in rows] == ["ST", "BM", "CM", "RT", "PR", "TB"]


def test_oracle_lattice_equals_table1_brute_force():
    rows, _ = _table1()
    lat = _lattice_from_table1(rows)
    assert sorted(_mask(s) for s in lat) == sorted(oracle.valid_ocs())
    assert len(lat) == 30
    # every subset of the lattice is closed under dropping RT/PR/BM/CM/TB
    for s in lat:
        for a in s - {"ST"}:
            assert (s - {a}) in lat


def test_paper_tb_names():
    rows, extra = _table1()
    lat = _lattice_from_table1(rows)
    tb_no_st = sorted(oracle.oc_name(_mask(s)) for s in lat if "TB" in s and "ST" not in s)
    assert tb_no_st == sorted(extra["names_tb_without_st"])


def test_library_lattice_and_names_equal_table1():
    import paper_conf_ipps_sunlyjlq22_b200 as sm
    rows, extra = _table1()
    lat = _lattice_from_table1(rows)
    ids = sorted(sm.oc_list())
    assert ids == sorted(_mask(s) for s in lat)
    for n in extra["names_tb_without_st"]:
        assert n in {sm.oc_name(i) for i in ids}


def test_paper_workload_sizes_match_configs():
    """The paper's characterisation grids are bench workloads: C2/C4 run
    on 512^3, N2 (the 2-D label workload) on 8192^2; Algorithm-1 orders 1-4."""
    import stencil_inputs as si
    _, extra = _table1()
    g2 = tuple(int(x) for x in extra["grid_2d"])
    g3 = tuple(int(x) for x in extra["grid_3d"])
    assert si.CONFIGS["N2"]["dims"] == g2
    assert si.CONFIGS["C2"]["dims"] == g3 and si.CONFIGS["C4"]["dims"] == g3
    assert [int(x) for x in extra["orders"]] == [1, 2, 3, 4]
