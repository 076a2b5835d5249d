"""GPU parity of SURVEY 8(f) f2 (C16, approximate frequent values): ve_approx_topk against
vo_approx_topk, bit-exact, on cfg1, fuzz traces (every float width, NaN payloads,
mixed-type keys, invalid records) and a chunked + locally merged run."""
import numpy as np
import pytest

from gen import vegen as G
from oracle import oracle as O
from tests import workloads as W

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def _cmp(ctx, cfg, hobjs, recs, topk):
    nd, top = ctx.approx_topk()
    ond, otb, otc = O.approx_topk(cfg, hobjs, recs)
    assert np.array_equal(nd, ond)
    for k in range(len(nd)):
        m = int(min(nd[k], topk))
        assert np.array_equal(top[k, :m]["bits"], otb[k, :m]) and np.array_equal(top[k, :m]["count"], otc[k, :m]), k


@pytest.mark.parametrize("cfgc,seed,n,n_pcs,topk", [(G.CFG1, 1, 1 << 20, 16, 8), (G.FUZZ, 2, 65536, 64, 8),
                                                     (G.FUZZ, 4, 300001, 64, 3), (G.FUZZ, 9, 50000, 64, 64)])
def test_approx_parity(torch_cuda, cfgc, seed, n, n_pcs, topk):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    hobjs = W.host_objects(cfgc, 0, seed)
    recs = G.records_host(cfgc, 0, seed, 0, n)
    ctx = ve.Context(n_pcs=n_pcs, max_objects=max(len(hobjs), 1), topk=topk, hist_capacity=1 << 21)
    ctx.set_objects(W.device_objects(hobjs))
    ctx.analyze_records(W.device_records(recs), n)
    ctx.report()                                   # the report first (dense flush done) ...
    _cmp(ctx, O.make_config(n_pcs, topk=topk), hobjs, recs, topk)
    ctx.close()


def test_approx_without_report_and_merged(torch_cuda):
    """... or directly (ve_approx_topk flushes the dense counts itself); two contexts merged locally."""
    from paper_conf_asplos_zhouhmm022_b200 import ve
    seed, n = 6, 120000
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    recs = G.records_host(G.FUZZ, 0, seed, 0, n)
    a = ve.Context(n_pcs=64, max_objects=8, hist_capacity=1 << 21)
    b = ve.Context(n_pcs=64, max_objects=8, hist_capacity=1 << 21)
    dobjs = W.device_objects(hobjs)
    a.set_objects(dobjs)
    b.set_objects(dobjs)
    d = W.device_records(recs)
    a.analyze_records(d[:50000 * 24], 50000)
    b.analyze_records(d[50000 * 24:], n - 50000)
    a.merge(b)
    _cmp(a, O.make_config(64), hobjs, recs, 8)
    a.close()
    b.close()
