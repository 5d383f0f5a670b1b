"""Dataset rows ("each parameter setting and its
corresponding execution time are also stored in the stencil dataset"): the
resumable JSONL writer. CPU only -- rows are synthetic here; the GPU test of
the rows themselves is tests/test_gpu_parity.py::test_sweep_rows."""
import json
import math

from paper_conf_ipps_sunlyjlq22_b200 import dataset


def _block(sid, n_oc=3, k=2):
    rows = [{"stencil_id": sid, "kind": "setting", "oc": o, "setting": s, "time_ms": 1.0 + o + s}
            for o in range(n_oc) for s in range(k)]
    rows.append({"stencil_id": sid, "kind": "label", "best_oc": 0,
                 "oc_times_ms": {"base": 1.0, "ST": None}})
    return rows


def test_resume_cuts_torn_tail(tmp_path):
    p = str(tmp_path / "ds.jsonl")
    dataset.append_rows(p, _block("a"))
    dataset.append_rows(p, _block("b"))
    good = open(p, "rb").read()
    # an interrupted third stencil: two complete setting rows and a torn line
    with open(p, "a") as f:
        for r in _block("c")[:2]:
            f.write(json.dumps(r) + "\n")
        f.write(json.dumps(_block("c")[2])[:17])
    assert dataset.done_ids(p) == {"a", "b"}
    assert dataset.resume(p) == {"a", "b"}
    assert open(p, "rb").read() == good          # back to the end of b's label line
    dataset.append_rows(p, _block("c"))
    lines = [json.loads(x) for x in open(p)]
    assert [x["stencil_id"] for x in lines if x["kind"] == "label"] == ["a", "b", "c"]
    for sid in "abc":                             # no duplicated setting rows
        assert sum(1 for x in lines if x["stencil_id"] == sid and x["kind"] == "setting") == 6
    ids, names, m = dataset.load_matrix(p)
    assert ids == ["a", "b", "c"] and m.shape == (3, len(names))
    assert m[0, names.index("base")] == 1.0 and math.isinf(m[0, names.index("ST")])


def test_resume_missing_and_clean_files(tmp_path):
    p = str(tmp_path / "none.jsonl")
    assert dataset.resume(p) == set()
    dataset.append_rows(p, _block("x"))
    before = open(p, "rb").read()
    assert dataset.resume(p) == {"x"}
    assert open(p, "rb").read() == before
    # orphaned setting rows after the last label (label never written) are dropped
    with open(p, "a") as f:
        f.write(json.dumps(_block("y")[0]) + "\n")
    assert dataset.resume(p) == {"x"} and open(p, "rb").read() == before
