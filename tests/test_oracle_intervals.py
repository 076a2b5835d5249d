"""Oracle pins of C13-C15 (PAPER.md 6.1).

The oracle merges by sort + sweep (oracle/ve_oracle.c).  It is pinned here by
methods that share nothing with it:
  * brute-force byte coverage on a small universe (the union, then its runs),
  * a literal transcription of Figure 4's nine steps: sort the
    (address, is_end) end points with ends after starts, +1/-1 markers, prefix
    scan, start flags, scan, end flags, scan, scatter -- with half-open ends
    (end + 1) so that "adjacent" intervals merge,
  * closed forms (cfg1 covers its object exactly once: one interval),
  * hand-worked copy plans (Figure 5).
"""
import numpy as np
import pytest

from gen import vegen as G
from oracle import oracle as O
from tests.helpers import meta, records, U, F, BF

IV = O.INTERVAL_DTYPE


def ivs(pairs):
    a = np.zeros(len(pairs), dtype=IV)
    for i, (s, e) in enumerate(pairs):
        a[i] = (s, e)
    return a


def runs_of(covered):
    """maximal runs of True in a boolean array -> list of (start, end) inclusive"""
    out, i, n = [], 0, len(covered)
    while i < n:
        if covered[i]:
            j = i
            while j + 1 < n and covered[j + 1]:
                j += 1
            out.append((i, j))
            i = j + 1
        else:
            i += 1
    return out


def brute_merge(pairs, universe):
    cov = np.zeros(universe, dtype=bool)
    for s, e in pairs:
        if s <= e:
            cov[s:e + 1] = True
    return runs_of(cov)


def figure4_merge(pairs):
    """Figure 4, steps 1-9, with half-open ends so adjacency merges."""
    pts = []
    for s, e in pairs:
        if s <= e:
            pts.append((s, 0))          # start
            pts.append((e + 1, 1))      # end (half-open), sorted after a start at the same address
    if not pts:
        return []
    pts.sort()                                              # 1: lexicographic (address, is_end)
    markers = np.array([1 if t == 0 else -1 for _, t in pts])   # 2
    ps = np.cumsum(markers)                                 # 3: prefix scan
    sflag = np.array([1 if (ps[i] == 1 and pts[i][1] == 0) else 0 for i in range(len(pts))])  # 4
    sidx = np.cumsum(sflag) - 1                             # 5: output indices of starts
    eflag = np.array([1 if (ps[i] == 0 and pts[i][1] == 1) else 0 for i in range(len(pts))])  # 6
    eidx = np.cumsum(eflag) - 1                             # 7
    k = int(sflag.sum())
    starts, ends = [0] * k, [0] * k
    for i in range(len(pts)):
        if sflag[i]:
            starts[sidx[i]] = pts[i][0]                     # 8
        if eflag[i]:
            ends[eidx[i]] = pts[i][0] - 1                   # 9 (back to inclusive)
    return list(zip(starts, ends))


def as_pairs(a):
    return [(int(x["start"]), int(x["end"])) for x in a]


@pytest.mark.parametrize("seed", range(12))
def test_merge_matches_brute_force_and_figure4(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(0, 60))
    U_ = 160
    s = rng.integers(0, U_, n)
    ln = rng.integers(-3, 12, n)               # negative lengths: empty intervals (start > end)
    pairs = [(int(a), int(min(U_ - 1, max(0, a + b)))) if b >= 0 else (int(a), int(a) - 1 if a > 0 else 0)
             for a, b in zip(s, ln)]
    pairs = [(a, e) for a, e in pairs if e >= 0]
    got = as_pairs(O.interval_merge(ivs(pairs)))
    assert got == brute_merge(pairs, U_)
    assert got == figure4_merge(pairs)


def test_merge_edge_cases():
    assert as_pairs(O.interval_merge(ivs([]))) == []
    assert as_pairs(O.interval_merge(ivs([(5, 4)]))) == []                          # empty only
    assert as_pairs(O.interval_merge(ivs([(0, 0), (1, 1), (2, 2)]))) == [(0, 2)]    # adjacent chain
    assert as_pairs(O.interval_merge(ivs([(0, 0), (2, 2)]))) == [(0, 0), (2, 2)]    # a 1-byte gap stays
    assert as_pairs(O.interval_merge(ivs([(10, 20), (12, 15)]))) == [(10, 20)]      # containment
    top = (1 << 64) - 1
    assert as_pairs(O.interval_merge(ivs([(top - 3, top), (5, 9), (top, top)]))) == [(5, 9), (top - 3, top)]
    assert as_pairs(O.interval_merge(ivs([(0, top), (7, 8)]))) == [(0, top)]
    # order of the input does not matter
    p = [(30, 40), (0, 3), (41, 41), (4, 9), (100, 120), (50, 60)]
    assert as_pairs(O.interval_merge(ivs(p))) == as_pairs(O.interval_merge(ivs(p[::-1]))) == \
        [(0, 9), (30, 41), (50, 60), (100, 120)]


@pytest.mark.parametrize("seed", range(6))
def test_record_intervals_brute_force(seed):
    """C14: byte coverage of the valid global-space records; invalid and shared ones excluded."""
    rng = np.random.default_rng(100 + seed)
    rows, cov = [], np.zeros(512, dtype=bool)
    for _ in range(int(rng.integers(1, 200))):
        w = int(rng.choice([1, 2, 4, 8]))
        a = int(rng.integers(0, 512 - 8))
        kind = U if w == 1 else int(rng.choice([U, F]))
        shared = int(rng.random() < 0.15)
        bad = rng.random() < 0.15
        pc = 99 if bad else int(rng.integers(0, 4))          # pc >= n_pcs: invalid
        rows.append((a, 0, pc, meta(w, kind, int(rng.random() < 0.5), shared)))
        if not bad and not shared:
            cov[a:a + w] = True
    rows.append((3, 0, 0, meta(2, BF) | (1 << 7)))               # reserved meta bit: invalid
    got = as_pairs(O.record_intervals(4, records(rows)))
    assert got == runs_of(cov)


def test_record_intervals_cfg1_closed_form():
    """cfg1: 16 PCs x 65,536 4-byte elements cover the 4 MiB object exactly: one interval."""
    recs = G.records_host(G.CFG1, 0, 1, 0, 1 << 20)
    o = G.objects(G.CFG1)[0]
    assert as_pairs(O.record_intervals(16, recs)) == [(o["base"], o["base"] + o["size"] - 1)]


def test_copy_plan_hand_worked():
    """Figure 5: clipping, segment vs min-max choice (R3, R4)."""
    objs = [{"base": 100, "size": 100, "id": 0, "elem_width": 1, "pre": None, "post": None},
            {"base": 300, "size": 50, "id": 1, "elem_width": 1, "pre": None, "post": None},
            {"base": 200, "size": 10, "id": 2, "elem_width": 4, "pre": None, "post": None}]
    merged = O.interval_merge(ivs([(90, 104), (110, 110), (150, 160), (195, 230), (300, 349)]))
    p = O.plan_copies(objs, merged, seg_max=32, dense_pct=50)
    # object 0 = [100, 199]: clips [100,104] [110,110] [150,160] [195,199]
    assert (int(p[0]["n_segments"]), int(p[0]["accessed_bytes"]), int(p[0]["lo"]), int(p[0]["hi"])) == (4, 22, 100, 199)
    assert int(p[0]["minmax_bytes"]) == 100 and int(p[0]["direct_bytes"]) == 100
    assert p[0]["choice"] == O.COPY_SEGMENT                      # 22% < 50% and 4 <= 32
    # object 2 = [200, 209] lies inside [195, 230]: one dense segment -> min-max
    assert (int(p[2]["n_segments"]), int(p[2]["accessed_bytes"]), int(p[2]["lo"]), int(p[2]["hi"])) == (1, 10, 200, 209)
    assert p[2]["choice"] == O.COPY_MINMAX
    # object 1 fully covered
    assert int(p[1]["accessed_bytes"]) == 50 and p[1]["choice"] == O.COPY_MINMAX
    assert O.plan_copies(objs, merged, seg_max=3)[0]["choice"] == O.COPY_MINMAX      # too many intervals
    assert O.plan_copies(objs, merged, dense_pct=20)[0]["choice"] == O.COPY_MINMAX   # 22% is dense at T=20%
    none = O.plan_copies(objs, O.interval_merge(ivs([(0, 50)])))
    assert all(x["choice"] == O.COPY_NONE and x["n_segments"] == 0 and x["minmax_bytes"] == 0 for x in none)


@pytest.mark.parametrize("seed", range(4))
def test_copy_plan_brute_force(seed):
    rng = np.random.default_rng(200 + seed)
    objs, base = [], 0
    for i in range(5):
        base += int(rng.integers(0, 20))
        size = int(rng.integers(1, 60))
        objs.append({"base": base, "size": size, "id": (i * 3) % 5, "elem_width": 1, "pre": None, "post": None})
        base += size
    pairs = [(int(a), int(a + rng.integers(0, 15))) for a in rng.integers(0, base + 10, 25)]
    merged = O.interval_merge(ivs(pairs))
    cov = np.zeros(base + 40, dtype=bool)
    for s, e in pairs:
        cov[s:e + 1] = True
    plan = O.plan_copies(objs, merged, seg_max=3, dense_pct=40)
    for o in objs:
        c = cov[o["base"]:o["base"] + o["size"]]
        r = runs_of(c)
        p = plan[o["id"]]
        assert int(p["n_segments"]) == len(r) and int(p["accessed_bytes"]) == int(c.sum())
        if r:
            lo, hi = o["base"] + r[0][0], o["base"] + r[-1][1]
            assert (int(p["lo"]), int(p["hi"])) == (lo, hi)
            sparse = 100 * int(c.sum()) < 40 * (hi - lo + 1)
            assert p["choice"] == (O.COPY_SEGMENT if sparse and len(r) <= 3 else O.COPY_MINMAX)
        else:
            assert p["choice"] == O.COPY_NONE
