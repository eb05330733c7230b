"""Independent decoder of the DASP packed format (DESIGN.md §4 FORMAT) — test code only.

It inverts the layout and returns, for every original row, the list of its (col, value-bits)
in slot order, plus every pad it saw.  ``check_roundtrip`` then requires that the decoded
rows equal the CSR rows exactly (same order; pin P6 of SURVEY.md §8(c)): every nonzero is
recovered exactly once, in CSR order, and every pad is exactly (+0, col -1).
"""
from __future__ import annotations

import numpy as np

PAD = -1


def params(dtype):
    if dtype in ("f64", "f32"):
        return dict(K=4, BE=32, EPL=1, G=64, UG=4, CW=4)
    return dict(K=8, BE=64, EPL=2, G=128, UG=4, CW=4)


def _bits(vals):
    return vals.view({8: np.uint64, 4: np.uint32, 2: np.uint16}[vals.dtype.itemsize])


def decode(F, get, dtype):
    """F: counts dict; get(name) -> typed numpy array.  Returns (rows: dict row -> list[(col, bits)], pads)."""
    p = params(dtype)
    K, BE, EPL, G, CW = p["K"], p["BE"], p["EPL"], p["G"], p["CW"]
    rows = {}
    pads = []

    def emit(row, c, v):
        rows.setdefault(int(row), []).append((int(c), int(v)))

    # long: each row's groups hold its elements then trailing pads; every other slot is a pad
    lv, lc, gp, lo = _bits(get("long_val")), get("long_col"), get("group_ptr"), get("long_out")
    assert len(lv) == F["n_groups_padded"] * G
    covered = np.zeros(len(lc), dtype=bool)
    for r in range(F["row_long"]):
        seg_c = lc[gp[r] * G: gp[r + 1] * G]
        seg_v = lv[gp[r] * G: gp[r + 1] * G]
        covered[gp[r] * G: gp[r + 1] * G] = True
        real = seg_c != PAD
        nreal = int(real.sum())
        assert real[:nreal].all(), "long pads must trail the row"
        for c, v in zip(seg_c[:nreal], seg_v[:nreal]):
            emit(lo[r], c, v)
        pads += list(zip(seg_c[nreal:], seg_v[nreal:]))
    pads += list(zip(lc[~covered], lv[~covered]))
    assert (lc[~covered] == PAD).all()

    # medium: regular chunks, then irregular tails
    rv, rc, rbp = _bits(get("reg_val")), get("reg_col"), get("rb_ptr")
    iv, ic, ip, mo = _bits(get("irr_val")), get("irr_col"), get("irr_ptr"), get("med_out")
    for rb in range(F["nrb"]):
        nreg = (rbp[rb + 1] - rbp[rb]) // BE
        assert (rbp[rb + 1] - rbp[rb]) % BE == 0
        slots = {g: {} for g in range(8)}
        for b in range(nreg):
            c, jb = divmod(b, CW)
            w = min(CW, nreg - c * CW)
            base = rbp[rb] + c * CW * BE
            for lane in range(32):
                g, t = lane >> 2, lane & 3
                for e in range(EPL):
                    slot = K * b + (t if EPL == 1 else 2 * t + e)
                    # R18: full chunks lane-interleaved, the ragged last chunk block by block
                    at = base + (lane * w * EPL + jb * EPL + e if w == CW else jb * BE + lane * EPL + e)
                    slots[g][slot] = (rc[at], rv[at])
        for g in range(8):
            i = rb * 8 + g
            row = mo[i]
            seq = [slots[g][s] for s in sorted(slots[g])]
            real = [(c, v) for c, v in seq if c != PAD]
            assert all(c != PAD for c, _ in seq[:len(real)]), "regular pads must trail"
            pads += [(c, v) for c, v in seq if c == PAD]
            tail = list(zip(ic[ip[i]:ip[i + 1]], iv[ip[i]:ip[i + 1]]))
            if row < 0:
                assert not real and not tail
                continue
            if tail:
                assert len(real) == K * nreg, "irregular tail only after full regular slots"
            for c, v in real + tail:
                emit(row, c, v)
            rows.setdefault(int(row), [])

    # short tiles, panel by panel: [1&3][len4][2&2][singles] per panel
    sv, sc, so = _bits(get("short_val")), get("short_col"), get("short_out")
    panels = get("panels").reshape(-1, 12)
    for pn in panels:
        tile0, t13, t4, t22, ts, out0 = (int(v) for v in pn[6:12])
        for cat, ntl in enumerate([t13, t4, t22]):
            two = cat != 1
            for tl in range(ntl):
                grid = {}
                for lane in range(32):
                    g, t = lane >> 2, lane & 3
                    for j in range(4):
                        if dtype in ("f64", "f32"):
                            r, c = 8 * j + g, t
                        else:
                            r = 8 * ((t >> 1) + (0 if j < 2 else 2)) + g
                            c = 2 * (t & 1) + (j & 1)
                        at = (tile0 + tl) * 128 + lane * 4 + j
                        grid[(r, c)] = (sc[at], sv[at])
                for r in range(32):
                    cells = [grid[(r, c)] for c in range(4)]
                    if two:
                        o = out0 + tl * 64 + 16 * (r // 8) + (r % 8)
                        ra, rb_ = so[o], so[o + 8]
                        split = 1 if cat == 0 else 2
                        segs = [(ra, cells[:split]), (rb_, cells[split:])]
                    else:
                        segs = [(so[out0 + tl * 32 + r], cells)]
                    for row, seg in segs:
                        real = [(c, v) for c, v in seg if c != PAD]
                        assert all(c != PAD for c, _ in seg[:len(real)])
                        pads += [(c, v) for c, v in seg if c == PAD]
                        if row < 0:
                            assert not real
                            continue
                        for c, v in real:
                            emit(row, c, v)
            tile0 += ntl
            out0 += ntl * (64 if two else 32)
        for q in range(ts * 128):
            at = tile0 * 128 + q
            row = so[out0 + q]
            if row < 0:
                assert sc[at] == PAD
                pads.append((sc[at], sv[at]))
            else:
                emit(row, sc[at], sv[at])

    for e in get("empty_rows"):
        assert int(e) not in rows
        rows[int(e)] = []
    return rows, pads


def check_roundtrip(A, F, get, dtype):
    rows, pads = decode(F, get, dtype)
    for c, v in pads:
        assert c == PAD and v == 0, "pads must be exactly (+0, -1)"
    assert sorted(rows) == list(range(A.m)), "every row exactly once"
    vals = {"f64": A.val, "f32": A.val.astype(np.float32), "f16": A.val.astype(np.float16)}[dtype]
    bits = _bits(np.ascontiguousarray(vals))
    for i in range(A.m):
        a, b = A.row_ptr[i], A.row_ptr[i + 1]
        want = list(zip(A.col[a:b].tolist(), bits[a:b].tolist()))
        assert rows[i] == want, f"row {i}"
    return len(pads)
