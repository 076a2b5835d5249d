"""Pins of C22 (approximate structured: C21 over Def 3.8's truncated values, R11) and C23
(structured with <= eps outliers: the interior-anchor line, R12) against hand-fixed cases
and brute force with exact rational arithmetic (fractions.Fraction) on tiny traces."""
from fractions import Fraction
import itertools
import math

import numpy as np
import pytest

from oracle import oracle as O
from tests.test_oracle_dyadic import BASE, REC, brute, exact, meta

K = 7                                                     # Q6: default mantissa bits


def trunc_bits(bits, kind, w):
    """Def 3.8 / C7 truncation written out: clear the low m - K mantissa bits of a float"""
    if kind < 2:
        return int(bits)
    m = 7 if kind == 3 else {2: 10, 4: 23, 8: 52}[w]
    return int(bits) if K >= m else int(bits) & ~((1 << (m - K)) - 1)


def recs_of(rows):
    a = np.zeros(len(rows), dtype=REC)
    for i, (x, b, pc, m) in enumerate(rows):
        a[i] = (x, b, pc, m)
    return a


def f32(x):
    return int(np.array([x], dtype=np.float32).view(np.uint32)[0])


def f64(x):
    return int(np.array([x], dtype=np.float64).view(np.uint64)[0])


def _fit(fn, rows, n_pcs=1, **kw):
    objs = [{"base": BASE, "size": 1 << 20, "id": 0, "elem_width": 8, "pre": None, "post": None}]
    return fn(O.make_config(n_pcs), objs, recs_of(rows), **kw)


# ---------------------------------------------------------------------------- C22
def test_c22_noisy_ramp_is_approximately_structured():
    """f32 y_i = 1 + i/8 plus one ulp of noise on odd i: the exact fit fails, the truncated one is a line
    through (x_0, 1) and (x_31, 1 + 31/8) (scale: the ramp's 3 fractional bits)"""
    rows = []
    for i in range(32):
        b = f32(1 + i / 8) + (i & 1)
        rows.append((BASE + 4 * i, b, 0, meta(2, 2)))
    d = _fit(O.dyadic_fit, rows)
    t = _fit(O.dyadic_fit_trunc, rows)
    assert d[0]["state"] == 3
    assert t[0]["state"] == 2 and t[0]["scale"] == 3
    assert (t[0]["px"], t[0]["qx"]) == (BASE, BASE + 4 * 31)
    assert (t[0]["py"], t[0]["qy"]) == (8, 8 + 31)


def test_c22_equals_c21_on_integers_and_on_short_mantissas():
    """integer records are not truncated; floats with <= K significant mantissa bits are unchanged"""
    rows = [(BASE + 8 * i, (3 * i + 5) & 0xFFFFFFFF, 0, meta(2, 1)) for i in range(20)]
    rows += [(BASE + 0x1000 + 8 * i, f64(2.0 + 0.5 * i), 1, meta(3, 2)) for i in range(20)]
    a, b = _fit(O.dyadic_fit, rows, n_pcs=2), _fit(O.dyadic_fit_trunc, rows, n_pcs=2)
    assert a.tobytes() == b.tobytes()


@pytest.mark.parametrize("seed", range(6))
def test_c22_brute_force(seed):
    rng = np.random.default_rng(100 + seed)
    pool = [1.0, 1.5, 2.0, 3.25, -0.75, 1.0 + 2 ** -20, 2.0 - 2 ** -18, 0.1, float("nan"), 1024.0]
    rows = []
    for i in range(int(rng.integers(1, 9))):
        kind, w = [(2, 4), (2, 8), (2, 2), (3, 2)][int(rng.integers(0, 4))]
        v = pool[int(rng.integers(0, len(pool) - (0 if seed % 3 == 0 else 1)))]
        if kind == 3:
            b = f32(v) >> 16
        elif w == 2:
            b = int(np.array([v], dtype=np.float16).view(np.uint16)[0])
        elif w == 4:
            b = f32(v)
        else:
            b = f64(v)
        rows.append((BASE + 8 * int(rng.integers(0, 6)), b, 0, meta({2: 1, 4: 2, 8: 3}[w], kind)))
    got = _fit(O.dyadic_fit_trunc, rows)[0]
    pts = []
    for x, b, _, m in rows:
        kind, w = (m >> 2) & 3, 1 << (m & 3)
        v = exact(b, kind, w)                          # a NaN / inf record fails the key
        pts.append((x, None if v is None else exact(trunc_bits(b, kind, w), kind, w)))
    want = brute(pts)
    assert tuple(int(got[f]) for f in ("state", "scale", "px", "qx", "py", "qy")) == want


# ---------------------------------------------------------------------------- C23
def test_c23_srad_clamped_boundary():
    """srad_v1's iN[i] = i - 1 with the clamped boundary iN[0] = 0 (Table 1): the exact
    fit fails at the boundary element, the interior line holds every other point (n_off = 1)"""
    N = 64
    rows = [(BASE + 4 * i, (i - 1 if i > 0 else 0) & 0xFFFFFFFF, 0, meta(2, 1)) for i in range(N)]
    d = _fit(O.dyadic_fit, rows)
    o = _fit(O.outlier_fit, rows)[0]
    assert d[0]["state"] == 3
    assert o["state"] == 2 and (o["ax"], o["bx"]) == (BASE + 4, BASE + 4 * (N - 2))
    assert (o["ay"], o["by"]) == (0, N - 3)
    assert (o["n_off"], o["n"]) == (1, N)


def test_c23_degenerate_states():
    assert _fit(O.outlier_fit, [])[0]["state"] == 0
    three = [(BASE + 8 * i, i * i, 0, meta(2, 0)) for i in range(3)]            # 3 distinct x: no interior line
    o = _fit(O.outlier_fit, three)[0]
    assert o["state"] == 1 and o["n"] == 3
    nan = three + [(BASE + 64, 0x7FC00000, 0, meta(2, 2))]
    assert _fit(O.outlier_fit, nan)[0]["state"] == 3


def brute_outlier(points):
    """points: (x, exact value or None) -> (state, ax, bx, ay, by, n_off, n) from the definition"""
    if not points:
        return (0, 0, 0, 0, 0, 0, 0)
    if any(v is None for _, v in points):
        return (3, 0, 0, 0, 0, 0, 0)
    T = max(int(math.log2(v.denominator)) for _, v in points)
    if any(abs(v * (1 << T)) >= (1 << 62) for _, v in points):
        return (3, 0, 0, 0, 0, 0, 0)
    xs = sorted(set(x for x, _ in points))
    if len(xs) < 4:
        return (1, 0, 0, 0, 0, 0, len(points))
    ax, bx = xs[1], xs[-2]
    ay = min(v for x, v in points if x == ax)
    by = min(v for x, v in points if x == bx)
    off = sum(1 for x, v in points if (v - ay) * (bx - ax) != (by - ay) * (x - ax))
    return (2, ax, bx, int(ay * (1 << T)), int(by * (1 << T)), off, len(points))


@pytest.mark.parametrize("seed", range(8))
def test_c23_brute_force(seed):
    rng = np.random.default_rng(200 + seed)
    rows = []
    slope, icpt = int(rng.integers(-3, 4)), int(rng.integers(-10, 10))
    for i in range(int(rng.integers(1, 14))):
        xi = int(rng.integers(0, 9))
        y = slope * xi + icpt if rng.random() < 0.8 else int(rng.integers(-20, 20))
        if seed % 2:
            rows.append((BASE + 8 * xi, f64(y / 4.0), 0, meta(3, 2)))
        else:
            rows.append((BASE + 8 * xi, y & 0xFFFFFFFFFFFFFFFF, 0, meta(3, 1)))
    got = _fit(O.outlier_fit, rows)[0]
    pts = [(x, exact(b, (m >> 2) & 3, 1 << (m & 3))) for x, b, _, m in rows]
    want = brute_outlier(pts)
    assert tuple(int(got[f]) for f in ("state", "ax", "bx", "ay", "by", "n_off", "n")) == want


def test_c23_truncated_points():
    """flags & 1: the C22 truncation first -- a noisy f64 ramp with one clamped end is a line with one
    outlier only after truncation"""
    rows = [(BASE + 8 * i, f64(10.0 + i) + (3 if i % 3 == 0 else 0), 0, meta(3, 2)) for i in range(1, 40)]
    rows.append((BASE, f64(10.0 + 1), 0, meta(3, 2)))           # clamped boundary: x0 carries x1's value
    o_exact = _fit(O.outlier_fit, rows)[0]
    o_tr = _fit(O.outlier_fit, rows, flags=1)[0]
    assert o_exact["state"] == 2 and o_exact["n_off"] > 1
    assert o_tr["state"] == 2 and o_tr["n_off"] == 1 and o_tr["n"] == 40
