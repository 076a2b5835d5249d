"""Contexts are ordered by their own event and stream, never by device-wide synchronisation
(include/ve.h conventions; DESIGN section 5 "stream order"): several contexts driven from several
host threads on several streams at once, and one context fed from two streams without host
synchronisation, both give the oracle's report bit for bit."""
import threading

import pytest

from gen import vegen as G
from oracle import oracle as O
from tests import parity, workloads as W

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


@pytest.mark.parametrize("min_wpw", [0, 32])
def test_contexts_in_threads_match_oracle(torch_cuda, min_wpw):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    torch = torch_cuda
    cases = []
    for seed in (21, 22, 23, 24):
        hobjs = W.host_objects(G.FUZZ, 0, seed)
        recs = G.records_host(G.FUZZ, 0, seed, 0, 150001 + seed)
        cases.append((hobjs, recs, O.analyze(O.make_config(64), hobjs, recs)))
    bad, errors = [], []

    def work(i):
        try:
            hobjs, recs, (okeys, oglob, oobj) = cases[i]
            st = torch.cuda.Stream()
            ctx = ve.Context(n_pcs=64, max_objects=len(hobjs), hist_capacity=1 << 20, min_windows_per_warp=min_wpw)
            dobjs, drec = W.device_objects(hobjs), W.device_records(recs)
            torch.cuda.synchronize()
            for _ in range(3):                      # repeated epochs on one ctx: set_objects orders after the report
                ctx.set_objects(dobjs)
                ctx.analyze_records(drec, len(recs), stream=st.cuda_stream)
                rep = ctx.report()
                bad.extend(f"ctx {i}: " + m for m in parity.compare_with_oracle(rep, okeys, oglob, oobj))
                rep.close()
            ctx.close()
        except Exception as e:   # noqa: BLE001
            errors.append(repr(e))

    th = [threading.Thread(target=work, args=(i,)) for i in range(len(cases))]
    for t in th:
        t.start()
    for t in th:
        t.join()
    assert not errors, errors
    assert not bad, "\n".join(bad[:20])


def test_one_context_two_streams(torch_cuda):
    """Chunks of one trace analysed on two streams with no host synchronisation between the calls."""
    from paper_conf_asplos_zhouhmm022_b200 import ve
    torch = torch_cuda
    seed, n = 31, 400003
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    recs = G.records_host(G.FUZZ, 0, seed, 0, n)
    okeys, oglob, oobj = O.analyze(O.make_config(64), hobjs, recs)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    ctx = ve.Context(n_pcs=64, max_objects=len(hobjs), hist_capacity=1 << 20)
    ctx.set_objects(W.device_objects(hobjs))
    drec = W.device_records(recs)
    torch.cuda.synchronize()
    cuts = [0, 100000, 200001, 300000, n]
    for i, (a, b) in enumerate(zip(cuts[:-1], cuts[1:])):
        ctx.analyze_records(drec[a * 24:b * 24], b - a, stream=(s1 if i % 2 == 0 else s2).cuda_stream)
    rep = ctx.report()
    bad = parity.compare_with_oracle(rep, okeys, oglob, oobj)
    rep.close()
    ctx.close()
    assert not bad, "\n".join(bad[:20])
