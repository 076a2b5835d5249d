"""GPU parity of SURVEY 8(f) f3 (C17, LoadSpy temporal load redundancy in record order):
ve_temporal_loads against vo_temporal_loads on fuzz traces and hand-made traces, and the
full-size cfg2 gemm epoch (225.6 M records) against its closed form."""
import numpy as np
import pytest

from gen import vegen as G
from oracle import oracle as O
from tests import workloads as W
from tests.helpers import meta, records, obj, F

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


@pytest.mark.parametrize("seed,n", [(1, 4096), (2, 65536), (3, 300001)])
def test_temporal_fuzz_parity(torch_cuda, seed, n):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    recs = G.records_host(G.FUZZ, 0, seed, 0, n)
    # fold the addresses onto a few lines so that many loads repeat an address
    rng = np.random.default_rng(seed)
    recs = recs.copy()
    sel = rng.random(n) < 0.5
    recs["addr"][sel] = (recs["addr"][sel] & ~np.uint64(0xFFF)) | (recs["addr"][sel] & np.uint64(0x3C))
    ctx = ve.Context(n_pcs=64, max_objects=8)
    ctx.set_objects(W.device_objects(hobjs))
    got = ctx.temporal_loads(W.device_records(recs), n)
    want = O.temporal_loads(O.make_config(64), hobjs, recs)
    assert np.array_equal(got, want)
    assert int(want[:, 0].sum()) > 0
    ctx.close()


def test_temporal_hand_made(torch_cuda):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    A, C = 0x10000, 0x20000
    rows = [(A + 4 * e, 1000 + e, 0, meta(4, F)) for tile in range(5) for e in range(64)]
    rows += [(C, 0, 1, meta(4, F)), (C, 7, 2, meta(4, F, 1)), (C, 7, 1, meta(4, F)),
             (C, 0, 2, meta(4, F, 1)), (C, 0, 1, meta(4, F)), (C, 0, 1, meta(4, F))]
    recs = records(rows)
    hobjs = [obj(A, 256, 0, 4), obj(C, 4, 1, 4)]
    ctx = ve.Context(n_pcs=3, max_objects=2)
    ctx.set_objects(W.device_objects(hobjs))
    got = ctx.temporal_loads(W.device_records(recs), len(recs))
    assert np.array_equal(got, O.temporal_loads(O.make_config(3), hobjs, recs))
    assert got[0].tolist() == [256, 256] and got[1].tolist() == [3, 1]
    ctx.close()


def test_temporal_cfg2_full_size(torch_cuda):
    """Each weight is loaded once per (batch, N tile): 4 x 91 times; each workspace element once per
    (batch, M tile): 16 times; C once.  All re-reads see the same value (closed form)."""
    from paper_conf_asplos_zhouhmm022_b200 import ve
    torch = torch_cuda
    inf = G.info(G.CFG2, 1)
    n = inf["n_records"]
    recs = torch.empty(n * 24, dtype=torch.uint8, device="cuda")
    G.records_device(G.CFG2, 1, G.SEEDS[G.CFG2], 0, n, recs.data_ptr(), torch.cuda.current_stream().cuda_stream)
    ctx = ve.Context(n_pcs=inf["n_pcs"], max_objects=8)
    ctx.set_objects([dict(o, pre=None, post=None) for o in G.objects(G.CFG2, 1)])
    out = ctx.temporal_loads(recs, n)
    wa, wb = 256 * 1152, 1152 * 5776
    assert out[1].tolist() == [363 * wa, 363 * wa] and out[2].tolist() == [15 * wb, 15 * wb]
    assert out[3].tolist() == [0, 0] and out[0].tolist() == [0, 0] and out[4].tolist() == [0, 0]
    npc = inf["n_pcs"]
    assert out[npc + 0].tolist() == [363 * wa, 363 * wa] and out[npc + 1].tolist() == [15 * wb, 15 * wb]
    assert out[npc + 2].tolist() == [0, 0]
    ctx.close()


@pytest.mark.parametrize("cfg,epoch,seed,n", [(G.FUZZ, 0, 4, 300001), (G.scaled(G.CFG3, 6), 0, 3, None),
                                              (G.scaled(G.CFG4, 4), 1, 4, None)])
def test_temporal_pairs_parity(torch_cuda, cfg, epoch, seed, n):
    """f3 per (PC, object) (ve_temporal_loads_ex) against the oracle's pair table, bit-exact"""
    from paper_conf_asplos_zhouhmm022_b200 import ve
    inf = G.info(cfg, epoch)
    n = n or inf["n_records"]
    hobjs = W.host_objects(cfg, epoch, seed)
    recs = G.records_host(cfg, epoch, seed, 0, n)
    if cfg == G.FUZZ:                                  # repeats: fold addresses onto a few lines
        rng = np.random.default_rng(seed)
        recs = recs.copy()
        sel = rng.random(n) < 0.5
        recs["addr"][sel] = (recs["addr"][sel] & ~np.uint64(0xFFF)) | (recs["addr"][sel] & np.uint64(0x3C))
    ctx = ve.Context(n_pcs=inf["n_pcs"], max_objects=max(len(hobjs), 1))
    ctx.set_objects(W.device_objects(hobjs))
    keys, pairs = ctx.temporal_pairs(W.device_records(recs), n)
    ocfg = O.make_config(inf["n_pcs"])
    assert np.array_equal(keys, O.temporal_loads(ocfg, hobjs, recs))
    want = O.temporal_pairs(ocfg, hobjs, recs)
    assert np.array_equal(pairs, want)
    assert int(want[..., 0].sum()) > 0
    ctx.close()
