"""Pins of C21 (f2: dyadic-scaled exact linear fit, R10) against brute force with exact
rational arithmetic (fractions.Fraction): every float's value taken exactly through Python's
binary64, collinearity of EVERY triple of points checked, T / the 2^62 bound / the anchors
recomputed from their definitions."""
from fractions import Fraction
import itertools
import math

import numpy as np
import pytest

from oracle import oracle as O

REC = np.dtype([("addr", "<u8"), ("value", "<u8"), ("pc", "<u4"), ("meta", "<u4")])
BASE = 0x10000


def meta(lg, kind, st=0):
    return lg | (kind << 2) | (st << 4)


def exact(bits, kind, w):
    """exact value of the bits (None for NaN / inf)"""
    if kind == 0:
        return Fraction(int(bits))
    if kind == 1:
        b = int(bits)
        return Fraction(b - (1 << (8 * w)) if b >> (8 * w - 1) else b)
    if kind == 3:
        f = float(np.array([int(bits) << 16], dtype=np.uint32).view(np.float32)[0])
    elif w == 2:
        f = float(np.array([int(bits)], dtype=np.uint16).view(np.float16)[0])
    elif w == 4:
        f = float(np.array([int(bits)], dtype=np.uint32).view(np.float32)[0])
    else:
        f = float(np.array([int(bits)], dtype=np.uint64).view(np.float64)[0])
    return None if not math.isfinite(f) else Fraction(f)


def brute(points):
    """points: list of (x, value or None) -> (state, scale, px, qx, py, qy)"""
    if not points:
        return (0, 0, 0, 0, 0, 0)
    if any(v is None for _, v in points):
        return (3, 0, 0, 0, 0, 0)
    T = max(int(math.log2(v.denominator)) for _, v in points)       # denominators are powers of two
    Ys = [(x, v * (1 << T)) for x, v in points]
    assert all(Y.denominator == 1 for _, Y in Ys)
    if any(abs(Y) >= (1 << 62) for _, Y in Ys):
        return (3, 0, 0, 0, 0, 0)
    for (x1, y1), (x2, y2), (x3, y3) in itertools.combinations(Ys, 3):
        if (x2 - x1) * (y3 - y1) != (x3 - x1) * (y2 - y1):
            return (3, 0, 0, 0, 0, 0)
    xs = [x for x, _ in Ys]
    # a key with repeated x and different values fails the pairwise check through any third point,
    # or directly when only two points exist
    for (x1, y1), (x2, y2) in itertools.combinations(Ys, 2):
        if x1 == x2 and y1 != y2:
            return (3, 0, 0, 0, 0, 0)
    px, qx = min(xs), max(xs)
    py = min(Y for x, Y in Ys if x == px)
    qy = min(Y for x, Y in Ys if x == qx)
    return (1 if px == qx else 2, T, px, qx, int(py), int(qy))


def f32(v):
    return int(np.array([v], dtype=np.float32).view(np.uint32)[0])


def f64(v):
    return int(np.array([v], dtype=np.float64).view(np.uint64)[0])


def f16(v):
    return int(np.array([v], dtype=np.float16).view(np.uint16)[0])


def bf16(v):
    return f32(v) >> 16           # exact only for values with <= 8 significant bits


def roles(rng):
    """(name, [(x, bits)], meta) per PC: lines, near-lines, overflow, NaN, points, integer lines"""
    xs = BASE + 4 * np.arange(12, dtype=np.uint64)
    out = []
    out.append(("f32 ramp", [(x, f32(0.75 - 0.125 * i)) for i, x in enumerate(xs)], meta(2, 2)))
    bad = [(x, f32(0.75 - 0.125 * i)) for i, x in enumerate(xs)]
    bad[5] = (bad[5][0], bad[5][1] + 1)
    out.append(("f32 ramp, one ulp off", bad, meta(2, 2)))
    out.append(("f64 ramp k 2^-40", [(x, f64(3.0 + i * 2.0 ** -40)) for i, x in enumerate(xs)], meta(3, 2)))
    out.append(("f64 overflow 2^-60 vs 2^10", [(xs[0], f64(2.0 ** -60)), (xs[1], f64(1024.0))], meta(3, 2)))
    out.append(("f32 nan", [(xs[0], f32(1.0)), (xs[1], 0x7FC00000)], meta(2, 2)))
    out.append(("f32 inf", [(xs[0], 0x7F800000)], meta(2, 2)))
    out.append(("point", [(xs[3], f32(2.5)), (xs[3], f32(2.5))], meta(2, 2)))
    out.append(("point two values", [(xs[3], f32(2.5)), (xs[3], f32(-1.0))], meta(2, 2)))
    out.append(("f16 ramp", [(x, f16(-4.0 + 0.5 * i)) for i, x in enumerate(xs)], meta(1, 2)))
    out.append(("bf16 ramp", [(x, bf16(1.5 + 0.25 * i)) for i, x in enumerate(xs)], meta(1, 3)))
    out.append(("+0/-0 constant", [(x, 0x80000000 if i % 2 else 0) for i, x in enumerate(xs)], meta(2, 2)))
    out.append(("i32 line", [(x, (5 - 3 * i) & 0xFFFFFFFF) for i, x in enumerate(xs)], meta(2, 1)))
    out.append(("u64 huge", [(xs[0], 1 << 63), (xs[1], 0)], meta(3, 0)))
    out.append(("two x, repeated", [(xs[0], f32(1.0)), (xs[4], f32(2.0)), (xs[0], f32(3.0))], meta(2, 2)))
    pts = [(x, f32(float(rng.integers(-8, 8)) / 4)) for x in xs[:4]]
    out.append(("random quarters", pts, meta(2, 2)))
    out.append(("subnormal ramp", [(x, i + 1) for i, x in enumerate(xs)], meta(2, 2)))
    out.append(("f64 x-reversed order", [(x, f64(-2.0 * i + 0.5)) for i, x in reversed(list(enumerate(xs)))],
                meta(3, 2)))
    return out


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_dyadic_fit_brute_force(seed):
    rng = np.random.default_rng(seed)
    rs = roles(rng)
    rows = []
    for pc, (_, pts, m) in enumerate(rs):
        for x, b in pts:
            rows.append((int(x), int(b), pc, m))
    order = rng.permutation(len(rows))
    recs = np.array([rows[i] for i in order], dtype=REC)
    cfg = O.make_config(len(rs))
    got = O.dyadic_fit(cfg, [], recs)
    for pc, (name, pts, m) in enumerate(rs):
        kind, w = (m >> 2) & 3, 1 << (m & 3)
        want = brute([(int(x), exact(b, kind, w)) for x, b in pts])
        g = got[pc]
        assert (int(g["state"]), int(g["scale"]), int(g["px"]), int(g["qx"]), int(g["py"]), int(g["qy"])) == want, \
            name
    # the no-object key layout: PC keys then the SHARED key (empty here)
    assert len(got) == len(rs) + 1 and got[-1]["state"] == 0


def test_dyadic_fit_expected_states():
    """the states the recipe of each role fixes by hand (guards the brute force itself)"""
    rs = roles(np.random.default_rng(0))
    rows = [(int(x), int(b), pc, m) for pc, (_, pts, m) in enumerate(rs) for x, b in pts]
    got = O.dyadic_fit(O.make_config(len(rs)), [], np.array(rows, dtype=REC))
    want = {"f32 ramp": 2, "f32 ramp, one ulp off": 3, "f64 ramp k 2^-40": 2, "f64 overflow 2^-60 vs 2^10": 3,
            "f32 nan": 3, "f32 inf": 3, "point": 1, "point two values": 3, "f16 ramp": 2, "bf16 ramp": 2,
            "+0/-0 constant": 2, "i32 line": 2, "u64 huge": 3, "two x, repeated": 3, "subnormal ramp": 2,
            "f64 x-reversed order": 2}
    for pc, (name, _, _) in enumerate(rs):
        if name in want:
            assert int(got[pc]["state"]) == want[name], name
    i = [n for n, _, _ in rs].index("f32 ramp")
    assert int(got[i]["scale"]) == 3 and int(got[i]["py"]) == 6 and int(got[i]["qy"]) == 6 - 11   # 0.75*8, ...
    i = [n for n, _, _ in rs].index("f64 ramp k 2^-40")
    assert int(got[i]["scale"]) == 40


def test_dyadic_fit_object_keys():
    """object keys collect the records of their range; the integer-only case agrees with C8's line fit"""
    n = 64
    x = BASE + 4 * np.arange(n, dtype=np.uint64)
    recs = np.zeros(n, dtype=REC)
    recs["addr"] = x
    recs["value"] = [(7 * i + 3) & 0xFFFFFFFF for i in range(n)]
    recs["pc"] = np.arange(n) % 2
    recs["meta"] = meta(2, 1)
    objs = [{"base": BASE, "size": 4 * n, "id": 0, "elem_width": 4, "pre": None, "post": None}]
    cfg = O.make_config(2)
    got = O.dyadic_fit(cfg, objs, recs)
    keys, _, _ = O.analyze(cfg, objs, recs)
    for k in range(3):
        assert int(got[k]["state"]) == int(keys["line_state"][k]) == 2
        assert int(got[k]["px"]) == int(keys["p_x"][k]) and int(got[k]["qx"]) == int(keys["q_x"][k])
        assert int(got[k]["scale"]) == 0
