"""Golden fixtures (tests/golden/*.json): worked examples fixed by the paper's text, each file citing
the PAPER.md passage it restates (Figure 6, the long-row padding rule, the 0.75 regular-block
threshold, short-row piecing).  Every expected count, array and y value in a fixture is derived by
hand from that passage (the derivation is written next to it) -- none comes from the oracle or the
CUDA path.  Both the oracle's literal builder and the production host builder (host-only plan, no
GPU) must reproduce them, and the oracle's y must equal the closed-form sums exactly.  CPU only."""
import glob
import json
import os

import numpy as np
import pytest

import oracle
import synth
from paper_conf_sc_lu023_b200 import dasp
from tests.test_builder import COUNT_MAP

GOLDEN = sorted(glob.glob(os.path.join(os.path.dirname(__file__), "golden", "*.json")))


def _csr(rows, n):
    cols, vals, rp = [], [], [0]
    for r in rows:
        c = list(range(*r["range"])) if "range" in r else list(r["cols"])
        cols += c
        vals += [r["val"]] * len(c)
        rp.append(len(cols))
    return synth.CSR(len(rows), n, np.array(rp, dtype=np.int64), np.array(cols, dtype=np.int32),
                     np.array(vals, dtype=np.float64), "golden")


def _x(rule, n):
    assert rule == "j+1"
    return np.arange(1, n + 1, dtype=np.float64)


def _sections(fx):
    if "sections" in fx:
        for s in fx["sections"]:
            yield s["rows"], s["x"], s["expect_y"], [dict(s, max_len=256)]
    else:
        yield fx["rows"], fx["x"], fx["expect_y"], fx["cases"]


def _check_format(counts, get, case):
    for k, v in case.get("counts", {}).items():
        assert counts[k] == v, k
    for k, v in case.get("arrays", {}).items():
        assert get(k).tolist() == v, k
    for off, v in case.get("short_out_prefix", {}).items():
        so = get("short_out")
        assert so[int(off):int(off) + len(v)].tolist() == v, off
    lv = get("long_val")
    for r in case.get("long_row_layout", []):
        g0 = r["first_group"] * 64
        assert np.all(lv[g0:g0 + r["len"]] != 0), r
        assert np.all(lv[g0 + r["len"]:g0 + r["len"] + r["pads"]] == 0), r   # zeros appended after the row
        assert (r["len"] + r["pads"]) % 64 == 0


@pytest.mark.parametrize("path", GOLDEN, ids=[os.path.basename(p) for p in GOLDEN])
def test_golden_oracle(path):
    fx = json.load(open(path))
    assert fx["cite"].startswith("PAPER.md")
    for rows, xr, want_y, cases in _sections(fx):
        A = _csr(rows, fx["n"])
        y, _ = oracle.spmv_csr(A, _x(xr, A.n))
        assert y.tolist() == want_y                      # integer sums: exact
        for case in cases:
            F = oracle.build(A, fx["dtype"], max_len=case["max_len"])
            _check_format(F.counts, F.view, case)


@pytest.mark.parametrize("path", GOLDEN, ids=[os.path.basename(p) for p in GOLDEN])
def test_golden_host_builder(path):
    fx = json.load(open(path))
    for rows, _, _, cases in _sections(fx):
        A = _csr(rows, fx["n"])
        for case in cases:
            plan = dasp.dasp_plan_create(A.row_ptr, A.col, A.val, A.m, A.n, fx["dtype"], device=-1,
                                         max_len=case["max_len"])
            info = plan.info
            counts = {k: info[v] for k, v in COUNT_MAP.items()}

            def get(name):
                b = dasp.dasp_plan_copy_array(plan, name)
                if name.endswith("_val"):
                    return b.view(np.float64)
                return b.view(np.int64) if name in ("group_ptr", "rb_ptr", "irr_ptr", "panels") else b.view(np.int32)
            _check_format(counts, get, case)
            plan.destroy()
