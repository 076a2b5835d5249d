"""Pins for the two oracle outputs the round-1 pins left open (What's weak #3):

* vo_objstat.n_touched = #(W u L) (C10's "never accessed" complement, Q5; "addresses accessed
  by A") -- brute force over the records' element sets (Python sets), and cfg1's closed form (every
  element of the 4 MiB object is either stored (8 PCs) or loaded with its pre value (8 PCs)).
* C5 / C7: NaNs are excluded from ord_min / ord_max / trunc_min / trunc_max (raw_min / raw_max keep
  them) -- expected keys written as the bit constants C5 / C7 define for the listed numbers.

Expected values are constants or brute force, never a re-run of the oracle's formula.
"""
import numpy as np

from gen import vegen as G
from oracle import oracle as O
from tests.helpers import F, U, f32, f64, le_bytes, meta, obj, records

BASE = 0x7A0000000000


def _touched_brute(recs, base, size, ew, pre):
    """W = elements covered by stores fully inside; L = start elements of loads whose w bytes equal pre."""
    W, L = set(), set()
    for r in recs:
        a, v, m = int(r["addr"]), int(r["value"]), int(r["meta"])
        w = 1 << (m & 3)
        if not (base <= a and a + w <= base + size):
            continue
        off = a - base
        if (m >> 4) & 1:
            W.update(range(off // ew, (off + w - 1) // ew + 1))
        else:
            if int.from_bytes(pre[off:off + w].tobytes(), "little") == v:
                L.add(off // ew)
    return W, L


def test_n_touched_brute_force():
    rng = np.random.default_rng(7)
    ne, ew = 256, 4
    pre = le_bytes(rng.integers(0, 4, ne), ew)            # few values: loads hit eq_pre often
    rows = []
    for _ in range(600):
        e = int(rng.integers(0, ne + 4))                   # a few past the end (unmapped)
        st = int(rng.integers(0, 3) == 0)
        v = int(rng.integers(0, 4))
        rows.append((BASE + ew * e, v, 0, meta(4, U, store=st)))
    # a straddling store (no W bits, Q21) and a misaligned eq load (start element only)
    rows.append((BASE + ew * ne - 2, 0, 0, meta(4, U, store=1)))
    rows.append((BASE + 6, int.from_bytes(pre[6:10].tobytes(), "little"), 0, meta(4, U)))
    recs = records(rows)
    objs = [obj(BASE, ne * ew, 0, ew, pre=pre, post=pre.copy())]
    _, _, st = O.analyze(O.make_config(1), objs, recs)
    W, L = _touched_brute(recs, BASE, ne * ew, ew, pre)
    assert len(W) > 0 and len(L - W) > 0 and len(W - L) > 0   # the case separates W, L and W u L
    assert int(st[0]["n_written"]) == len(W)
    assert int(st[0]["n_loaded_eq"]) == len(L)
    assert int(st[0]["n_touched"]) == len(W | L)
    d = O.snapshot_diff(O.make_config(1), objs, recs, 0)
    assert int(d["n_untouched"]) == ne - len(W | L)


def test_n_touched_disjoint_and_overlap():
    """hand-fixed: stores on elements 0..9, eq loads on 5..19, non-eq loads on 30..35 -> |W u L| = 20"""
    ne, ew = 64, 4
    pre = le_bytes(range(ne), ew)
    rows = [(BASE + ew * e, 1000 + e, 0, meta(4, U, store=1)) for e in range(10)]
    rows += [(BASE + ew * e, e, 1, meta(4, U)) for e in range(5, 20)]
    rows += [(BASE + ew * e, e + 1, 1, meta(4, U)) for e in range(30, 36)]
    recs = records(rows)
    _, _, st = O.analyze(O.make_config(2), [obj(BASE, ne * ew, 0, ew, pre=pre, post=pre)], recs)
    assert (int(st[0]["n_written"]), int(st[0]["n_loaded_eq"]), int(st[0]["n_touched"])) == (10, 15, 20)


def test_n_touched_cfg1_closed_form():
    """cfg1: 8 store PCs and 8 load PCs (every load reads its pre value) each cover their own 65,536-element
    slice once, so W = 524,288, L = 524,288, W u L = all 1,048,576 elements."""
    objs = [dict(o, pre=G.snapshot_host(1, 0, 1, 0, 0), post=G.snapshot_host(1, 0, 1, 0, 1)) for o in G.objects(1)]
    recs = G.records_host(1, 0, 1, 0, 1 << 20)
    _, _, st = O.analyze(O.make_config(16), objs, recs)
    assert (int(st[0]["n_written"]), int(st[0]["n_loaded_eq"]), int(st[0]["n_touched"])) == \
        (524288, 524288, 1048576)
    # the first half only: PCs 0..15 each cover 32,768 of their slice -> W = L = 262,144, W u L = 524,288
    _, _, st = O.analyze(O.make_config(16), objs, recs[: 1 << 19])
    assert int(st[0]["n_touched"]) == 524288


# C5 orderable keys of f32 (sign clear: b | 2^31; sign set: ~b & mask) and C7 truncation (K = 7: clear
# the low 16 mantissa bits) written out for the numbers used below
ORD_F32 = {1.0: 0x3F800000 | 0x80000000, 2.0: 0x40000000 | 0x80000000, -3.0: ~0xC0400000 & 0xFFFFFFFF,
           1.5: 0x3FC00000 | 0x80000000}
TRUNC_F32 = {1.0: 0x3F800000, 2.0: 0x40000000, -3.0: 0xC0400000, 1.5: 0x3FC00000}


def test_nan_excluded_from_ord_and_trunc_f32():
    nan_pos, nan_neg, nan_payload = 0x7FC00000, 0xFFC00001, 0x7F800001
    vals = [f32(1.0), nan_pos, f32(2.0), nan_neg, f32(-3.0), nan_payload, f32(1.5) | 0x1234]
    # the last value is 1.5 plus low mantissa bits: same K=7 bucket as 1.5, ord above 1.5
    recs = records([(BASE + 4 * i, v, 0, meta(4, F)) for i, v in enumerate(vals)])
    k, _, _ = O.analyze(O.make_config(1), [obj(BASE, 64, 0, 4)], recs)
    k = k[0]
    assert int(k["n_nan"]) == 3
    assert int(k["raw_min"]) == f32(1.0) and int(k["raw_max"]) == nan_neg          # raw keeps NaNs
    assert int(k["ord_min"]) == ORD_F32[-3.0]                                      # not ~nan_neg's key
    assert int(k["ord_max"]) == ORD_F32[2.0]                                       # not nan_pos's key
    assert int(k["trunc_min"]) == TRUNC_F32[1.0] and int(k["trunc_max"]) == TRUNC_F32[-3.0]
    assert k["approx"] == 0                                                        # NaN present (C7)


def test_nan_only_key_keeps_identities():
    """a key whose only float values are NaN: ord / trunc min / max stay at their identities
    (min = 2^64 - 1, max = 0, DESIGN.md section 3 'Min/max identities')"""
    recs = records([(BASE + 8 * i, v, 0, meta(8, F)) for i, v in
                    enumerate([0x7FF8000000000000, 0xFFF0000000000001, 0x7FF0000000000002])])
    k, _, _ = O.analyze(O.make_config(1), [obj(BASE, 64, 0, 8)], recs)
    k = k[0]
    assert int(k["n_nan"]) == 3 and int(k["n_not_f32"]) == 3
    assert int(k["ord_min"]) == (1 << 64) - 1 and int(k["ord_max"]) == 0
    assert int(k["trunc_min"]) == (1 << 64) - 1 and int(k["trunc_max"]) == 0
    assert int(k["raw_min"]) == 0x7FF0000000000002 and int(k["raw_max"]) == 0xFFF0000000000001


def test_nan_excluded_f64_object_key():
    """the same on an object key mixing f64 loads and stores: ord of -0.5 is ~bits & mask (C5)"""
    vals = [f64(-0.5), 0x7FF8000000000000, f64(4.0), 0xFFF8000000000000]
    recs = records([(BASE + 8 * i, v, i % 2, meta(8, F, store=i % 2)) for i, v in enumerate(vals)])
    k, _, _ = O.analyze(O.make_config(2), [obj(BASE, 64, 0, 8)], recs)
    ko = k[2]                                                                      # object key 0
    assert int(ko["ord_min"]) == (~f64(-0.5)) & ((1 << 64) - 1)
    assert int(ko["ord_max"]) == f64(4.0) | (1 << 63)
    # K = 7 of f64 clears the low 45 mantissa bits; -0.5 and 4.0 have none set
    assert int(ko["trunc_min"]) == f64(4.0) and int(ko["trunc_max"]) == f64(-0.5)
