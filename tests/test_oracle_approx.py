"""Oracle pins of C16 (approximate frequent values = Def 3.3 over the
truncated values of Def 3.8).  Pinned by closed forms (cfg1 PCs
4, 5, 7; the paper's hotspot3D bucket), the NaN reading R5, the Q15 type rule,
and brute force over random floats of every width (truncation done independently with
numpy integer masks)."""
import collections
import struct

import numpy as np
import pytest

from gen import vegen as G
from oracle import oracle as O
from tests.helpers import meta, records, obj, F, BF, U, f32, f64


def _run(n_pcs, objs, rows, topk=8, K=7):
    cfg = O.make_config(n_pcs, topk=topk, mant_bits=K)
    return O.approx_topk(cfg, objs, records(rows) if isinstance(rows, list) else rows)


def test_cfg1_closed_forms():
    recs = G.records_host(G.CFG1, 0, 1, 0, 1 << 20)
    nd, tb, tc = O.approx_topk(O.make_config(16), [dict(o, pre=None, post=None) for o in G.objects(G.CFG1)], recs)
    # PC5: 1.0f + (e mod 4096) 2^-21 -> one bucket 1.0f (the approx single value of cfg1)
    assert nd[5] == 1 and tb[5, 0] == 0x3F800000 and tc[5, 0] == 65536
    # PC4: 1.0f except e mod 10 == 9 (random |v| < 1): the 1.0f bucket holds exactly the 58,982 ones
    assert tb[4, 0] == 0x3F800000 and tc[4, 0] == 58982
    # PC7: tenths 0.1 .. 1.0 stay 10 distinct buckets with the exact counts
    assert nd[7] == 10 and sorted(tc[7, :8].tolist() + [0]) [-8:] == sorted([6553, 6553, 6554, 6554, 6554, 6554, 6554, 6554])
    # integer PCs and the mixed-type object key have no approximate histogram
    assert nd[0] == nd[2] == nd[6] == 0 and nd[16] == 0


def test_hotspot_bucket_p7():
    """hotspot3D temperatures in one truncation bucket; 302.0 opens the next one."""
    base = 0x7f0000000000
    vals = [300.0 + k / 1024.0 for k in range(2048)]          # [300, 302)
    rows = [(base + 8 * i, f64(v), 0, meta(8, F)) for i, v in enumerate(vals)]
    rows += [(base + 8 * 3000, f64(302.0), 0, meta(8, F))]
    nd, tb, tc = _run(1, [obj(base, 8 * 4096, 0, 8)], rows)
    assert nd[0] == 2 and tb[0, 0] == f64(300.0) and tc[0, 0] == 2048 and tb[0, 1] == f64(302.0)


def test_nan_payloads_kept_and_mixed_types():
    rows = [(0x1000, 0x7FC00001, 0, meta(4, F)), (0x1004, 0x7FC00002, 0, meta(4, F)),
            (0x1008, f32(1.0), 0, meta(4, F)), (0x100C, f32(1.0000001), 0, meta(4, F)),
            (0x2000, f32(2.0), 1, meta(4, F)), (0x2004, 2, 1, meta(4, U))]       # PC1: mixed f32 / u32
    nd, tb, tc = _run(2, [], rows)
    assert nd[0] == 3                      # two NaN payloads stay apart; 1.0 and 1.0000001 share a bucket
    assert tb[0, 0] == f32(1.0) and tc[0, 0] == 2
    assert nd[1] == 0


def _trunc_np(bits, kind, w, K):
    m = 7 if kind == BF else {2: 10, 4: 23, 8: 52}[w]
    return bits if K >= m else bits & ~((1 << (m - K)) - 1)


def _is_nan(bits, kind, w):
    eb, mb = {(F, 2): (5, 10), (F, 4): (8, 23), (F, 8): (11, 52), (BF, 2): (8, 7)}[(kind, w)]
    return ((bits >> mb) & ((1 << eb) - 1)) == (1 << eb) - 1 and (bits & ((1 << mb) - 1)) != 0


@pytest.mark.parametrize("kind,w", [(F, 2), (F, 4), (F, 8), (BF, 2)])
@pytest.mark.parametrize("K", [0, 3, 7])
def test_brute_force(kind, w, K):
    rng = np.random.default_rng(w * 10 + K + kind)
    n = 3000
    nbits = 8 * w
    pool = rng.integers(0, 1 << min(nbits, 63), 64, dtype=np.uint64).tolist()
    pool += [0, 1 << (nbits - 1)]                                     # +0.0, -0.0
    pool += [((1 << (nbits - 1)) - 1)]                                # a NaN with every payload bit
    vals = [int(pool[i]) for i in rng.integers(0, len(pool), n)]
    rows = [(0x100000 + w * i, v, 0, meta(w, kind)) for i, v in enumerate(vals)]
    nd, tb, tc = _run(1, [], rows, topk=5, K=K)
    want = collections.Counter(v if _is_nan(v, kind, w) else _trunc_np(v, kind, w, K) for v in vals)
    order = sorted(want.items(), key=lambda kv: (-kv[1], kv[0]))[:5]
    assert nd[0] == len(want)
    assert [(int(tb[0, i]), int(tc[0, i])) for i in range(len(order))] == order
