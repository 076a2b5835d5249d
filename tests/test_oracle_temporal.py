"""Oracle pins of C17 (LoadSpy temporal load redundancy in record order,
Q1 / R6).  Pinned by an O(n^2) brute force that scans backwards for
each load's predecessor (a different method from the oracle's last-load table), by a
Darknet-style closed form (A re-read once per output tile), and by cfg1
(every element loaded once: nothing temporal)."""
import numpy as np
import pytest

from gen import vegen as G
from oracle import oracle as O
from tests.helpers import meta, records, obj, U, F


def brute(n_pcs, objs, rows):
    n_keys = n_pcs + len(objs) + 1
    out = np.zeros((n_keys, 2), dtype=np.uint64)
    def valid(r):
        a, v, pc, m = r
        w = 1 << (m & 3)
        kind = (m >> 2) & 3
        return not (m >> 6) and not (kind == 2 and w == 1) and not (kind == 3 and w != 2) and pc < n_pcs \
            and (w == 8 or v >> (8 * w) == 0) and a < (1 << 48)
    def is_load(r):
        return valid(r) and not (r[3] >> 4) & 1 and not (r[3] >> 5) & 1
    for i, r in enumerate(rows):
        if not is_load(r):
            continue
        prev = None
        for j in range(i - 1, -1, -1):
            if is_load(rows[j]) and rows[j][0] == r[0]:
                prev = rows[j]
                break
        if prev is None:
            continue
        red = int((prev[3] & 3) == (r[3] & 3) and prev[1] == r[1])
        keys = [r[2]]
        for o in objs:
            if o["base"] <= r[0] < o["base"] + o["size"]:
                keys.append(n_pcs + o["id"])
        for k in keys:
            out[k, 0] += 1
            out[k, 1] += red
    return out


@pytest.mark.parametrize("seed", range(8))
def test_brute_force(seed):
    rng = np.random.default_rng(seed)
    objs = [obj(0x1000, 64, 0, 4), obj(0x2000, 32, 1, 8)]
    addrs = [0x1000 + 4 * i for i in range(16)] + [0x2000 + 8 * i for i in range(4)] + [0x5000, 0x5004]
    rows = []
    for _ in range(int(rng.integers(1, 400))):
        a = int(rng.choice(addrs))
        w = int(rng.choice([4, 4, 4, 8, 2]))
        v = int(rng.integers(0, 3))                    # few values: many repeats
        st = int(rng.random() < 0.25)
        sh = int(rng.random() < 0.05)
        pc = int(rng.integers(0, 5)) if rng.random() > 0.05 else 9      # pc 9: invalid
        rows.append((a, v, pc, meta(w, U, st, sh)))
    got = O.temporal_loads(O.make_config(5), objs, records(rows))
    assert np.array_equal(got, brute(5, objs, rows))


def test_darknet_closed_form():
    """A[m][k] (64 elements) re-read by 5 output tiles: 4 x 64 temporal loads, all redundant.
    C: load 0; store 7; load 7 (temporal, not redundant: the last load read 0); store 0; load 0 (not
    redundant: the last load read 7); load 0 (redundant)."""
    A, C = 0x10000, 0x20000
    rows = []
    for tile in range(5):
        for e in range(64):
            rows.append((A + 4 * e, 1000 + e, 0, meta(4, F)))
    rows += [(C, 0, 1, meta(4, F)), (C, 7, 2, meta(4, F, 1)), (C, 7, 1, meta(4, F)),
             (C, 0, 2, meta(4, F, 1)), (C, 0, 1, meta(4, F)), (C, 0, 1, meta(4, F))]
    out = O.temporal_loads(O.make_config(3), [obj(A, 256, 0, 4), obj(C, 4, 1, 4)], records(rows))
    assert out[0].tolist() == [256, 256]               # PC0: (5 - 1) * 64, all the same values
    assert out[1].tolist() == [3, 1]                   # PC1: 7 after 0, 0 after 7, 0 after 0
    assert out[3].tolist() == [256, 256] and out[4].tolist() == [3, 1]


def test_cfg1_nothing_temporal():
    recs = G.records_host(G.CFG1, 0, 1, 0, 1 << 20)
    out = O.temporal_loads(O.make_config(16), [dict(o, pre=None, post=None) for o in G.objects(G.CFG1)], recs)
    assert int(out.sum()) == 0


def brute_pairs(n_pcs, objs, rows):
    """the O(n^2) backwards scan, counted per (pc, object of the first byte) -- column len(objs): none"""
    out = np.zeros((n_pcs, len(objs) + 1, 2), dtype=np.uint64)
    def valid(r):
        a, v, pc, m = r
        w = 1 << (m & 3)
        kind = (m >> 2) & 3
        return not (m >> 6) and not (kind == 2 and w == 1) and not (kind == 3 and w != 2) and pc < n_pcs \
            and (w == 8 or v >> (8 * w) == 0) and a < (1 << 48)
    def is_load(r):
        return valid(r) and not (r[3] >> 4) & 1 and not (r[3] >> 5) & 1
    for i, r in enumerate(rows):
        if not is_load(r):
            continue
        prev = next((rows[j] for j in range(i - 1, -1, -1) if is_load(rows[j]) and rows[j][0] == r[0]), None)
        if prev is None:
            continue
        col = next((o["id"] for o in objs if o["base"] <= r[0] < o["base"] + o["size"]), len(objs))
        out[r[2], col, 0] += 1
        out[r[2], col, 1] += int((prev[3] & 3) == (r[3] & 3) and prev[1] == r[1])
    return out


@pytest.mark.parametrize("seed", range(6))
def test_pairs_brute_force(seed):
    """f3 per (PC, object): the pair table against the backwards scan; its rows / columns sum to the
    per-PC / per-object keys of C17"""
    rng = np.random.default_rng(50 + seed)
    objs = [obj(0x1000, 64, 0, 4), obj(0x2000, 32, 1, 8)]
    addrs = [0x1000 + 4 * i for i in range(16)] + [0x2000 + 8 * i for i in range(4)] + [0x5000, 0x5004]
    rows = []
    for _ in range(int(rng.integers(1, 400))):
        a = int(rng.choice(addrs))
        rows.append((a, int(rng.integers(0, 3)), int(rng.integers(0, 5)), meta(int(rng.choice([4, 8, 2])), U,
                                                                            int(rng.random() < 0.25))))
    got = O.temporal_pairs(O.make_config(5), objs, records(rows))
    assert np.array_equal(got, brute_pairs(5, objs, rows))
    keys = O.temporal_loads(O.make_config(5), objs, records(rows))
    assert np.array_equal(got.sum(axis=1), keys[:5])                  # per PC
    assert np.array_equal(got[:, :2].sum(axis=0), keys[5:7])          # per object
