"""GPU parity: libve.so (sm_100a) against the CPU oracle, bit-exact, through
the C ABI.  Sizes span many CTAs/windows and ragged tails; adversarial fuzz
traces exercise every slow path."""
import numpy as np
import pytest

from gen import vegen as G
from gen import vegen as gen
from oracle import oracle as O
from tests import parity, workloads as W

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


from tests.gpu_run import _check, _run_gpu, _ve  # noqa: E402


def test_cfg1_parity(torch_cuda):
    hobjs = W.host_objects(G.CFG1, 0, 1)
    recs = G.records_host(G.CFG1, 0, 1, 0, 1 << 20)
    rep, okeys = _check(torch_cuda, 16, hobjs, recs)
    assert rep.keys["structured"][2] == 1 and rep.keys["approx"][5] == 1      # the cfg1 closed forms hold on GPU too


@pytest.mark.parametrize("seed,n", [(1, 4096), (2, 65536), (3, 100003), (4, 300001)])
def test_fuzz_parity(torch_cuda, seed, n):
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    recs = G.records_host(G.FUZZ, 0, seed, 0, n)
    _check(torch_cuda, 64, hobjs, recs)


def test_fuzz_parity_topk_variants(torch_cuda):
    hobjs = W.host_objects(G.FUZZ, 0, 9)
    recs = G.records_host(G.FUZZ, 0, 9, 0, 50000)
    for k in (1, 3, 64):
        _check(torch_cuda, 64, hobjs, recs, topk=k)


def test_chunk_and_permutation_invariance(torch_cuda):
    """I10 / C12: chunked calls and shuffled records give the same report."""
    seed, n = 5, 120007
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    recs = G.records_host(G.FUZZ, 0, seed, 0, n)
    cfg = O.make_config(64)
    okeys, oglob, oobj = O.analyze(cfg, hobjs, recs)
    rep, _ = _run_gpu(torch_cuda, 64, hobjs, recs, chunks=[1, 33, 1000, 1001, 50000, 99999])
    assert not parity.compare_with_oracle(rep, okeys, oglob, oobj)
    perm = np.random.default_rng(1).permutation(n)
    rep, _ = _run_gpu(torch_cuda, 64, hobjs, recs[perm])
    assert not parity.compare_with_oracle(rep, okeys, oglob, oobj)


def test_local_merge(torch_cuda):
    """ve_merge_stats(dst, src): merge(A, B) == analyze(A u B)."""
    ve = _ve()
    seed, n = 6, 80000
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    recs = G.records_host(G.FUZZ, 0, seed, 0, n)
    cfg = O.make_config(64)
    okeys, oglob, oobj = O.analyze(cfg, hobjs, recs)
    dobjs = W.device_objects(hobjs)
    drec = W.device_records(recs)
    a = ve.Context(n_pcs=64, max_objects=8, hist_capacity=1 << 20)
    b = ve.Context(n_pcs=64, max_objects=8, hist_capacity=1 << 20)
    a.set_objects(dobjs)
    b.set_objects(dobjs)
    a.analyze_records(drec[:30011 * 24], 30011)
    b.analyze_records(drec[30011 * 24:], n - 30011)
    a.merge(b)
    bad = parity.compare_with_oracle(a.report(), okeys, oglob, oobj)
    assert not bad, "\n".join(bad[:20])


def test_dedup_parity(torch_cuda):
    ve = _ve()
    seed, unit = 3, 4096
    n = 60
    objs, hpost = [], []
    for i in range(n):
        o = G.dedup_object(seed, i, unit)
        host = G.dedup_host(seed, i, unit)
        hpost.append(host)
        objs.append(o)
    # adversaries: an all-zero object and its copy, a one-byte flip of a random one, a NULL post
    hobjs = [dict(o, pre=None, post=hpost[i]) for i, o in enumerate(objs)]
    hobjs[7] = dict(hobjs[7], post=None)
    oracle_groups = O.object_dedup(hobjs)
    import torch
    dposts = [torch.from_numpy(h).cuda() if h is not None else None for h in [o["post"] for o in hobjs]]
    dobjs = [dict(o, post=dposts[i], pre=None) for i, o in enumerate(hobjs)]
    ctx = ve.Context(n_pcs=1, max_objects=1)
    g = ctx.object_dedup(dobjs)
    assert list(g) == list(oracle_groups)
    assert len(set(g)) < n                                      # duplicates exist in the set


def test_capacity_overflow_is_an_error(torch_cuda):
    ve = _ve()
    hobjs = W.host_objects(G.FUZZ, 0, 8)
    recs = G.records_host(G.FUZZ, 0, 8, 0, 200000)
    ctx = ve.Context(n_pcs=64, max_objects=8, hist_capacity=1024)
    ctx.set_objects(W.device_objects(hobjs))
    ctx.analyze_records(W.device_records(recs), len(recs))
    with pytest.raises(ve.VeError) as ei:
        ctx.report()
    assert ei.value.status == ve.ERR_CAPACITY
    with pytest.raises(ve.VeError) as ei:
        ctx.analyze_records(W.device_records(recs[:10]), 10)
    assert ei.value.status == ve.ERR_STATE
    ctx.reset()                                                 # clears the poison


def test_empty_and_tiny(torch_cuda):
    hobjs = W.host_objects(G.FUZZ, 0, 12)
    for n in (1, 2, 31, 32, 33):
        recs = G.records_host(G.FUZZ, 0, 12, 7, n)
        _check(torch_cuda, 64, hobjs, recs)


@pytest.mark.parametrize("G", [2, 3, 4])
def test_rank_merge_simulated(torch_cuda, G):
    """S12 across ranks, simulated on one GPU: G contexts analyze contiguous record chunks
    (as bench ranks do), ve_merge_group runs the NCCL algorithm (allreduce / allgather /
    hash-partitioned all-to-all of view entries + re-rank) with device copies; every
    context must report exactly the oracle's result over all records."""
    ve = _ve()
    seed, n = 13, 150001
    hobjs = W.host_objects(gen.FUZZ, 0, seed)
    recs = gen.records_host(gen.FUZZ, 0, seed, 0, n)
    cfg = O.make_config(64)
    okeys, oglob, oobj = O.analyze(cfg, hobjs, recs)
    dobjs = W.device_objects(hobjs)
    drec = W.device_records(recs)
    ctxs = []
    for r in range(G):
        lo, hi = ve.rank_chunk(n, r, G)
        c = ve.Context(n_pcs=64, max_objects=8, hist_capacity=1 << 20)
        c.set_objects(dobjs)
        c.analyze_records(drec[lo * 24:hi * 24], hi - lo)
        ctxs.append(c)
    ve.merge_group(ctxs)
    for c in ctxs:
        bad = parity.compare_with_oracle(c.report(), okeys, oglob, oobj)
        assert not bad, "\n".join(bad[:20])
    with pytest.raises(ve.VeError):                           # merged contexts refuse more records
        ctxs[0].analyze_records(drec[:24], 1)


def test_nccl_merge_single_rank(torch_cuda):
    """ve_merge_stats over a real (1-rank) NCCL communicator leaves the result exact."""
    ve = _ve()
    seed, n = 14, 90000
    hobjs = W.host_objects(gen.FUZZ, 0, seed)
    recs = gen.records_host(gen.FUZZ, 0, seed, 0, n)
    okeys, oglob, oobj = O.analyze(O.make_config(64), hobjs, recs)
    comm = ve.nccl_comm_init(ve.nccl_unique_id(), 0, 1)
    c = ve.Context(n_pcs=64, max_objects=8, hist_capacity=1 << 20)
    c.set_objects(W.device_objects(hobjs))
    c.analyze_records(W.device_records(recs), n)
    c.merge(comm=comm)
    bad = parity.compare_with_oracle(c.report(), okeys, oglob, oobj)
    assert not bad, "\n".join(bad[:20])


@pytest.mark.parametrize("budget", ["0", "70000", "300000"])
def test_dense_pool_exhausted_parity(torch_cuda, budget):
    """Dense counter arrays are allocated from one pool when a (pc, access type) first claims
    one; claims beyond the pool take the hash path.  Results must not depend on the pool size."""
    import os
    old = os.environ.get("VE_DENSE_BUDGET")
    os.environ["VE_DENSE_BUDGET"] = budget
    try:
        hobjs = W.host_objects(G.FUZZ, 0, 12)
        recs = G.records_host(G.FUZZ, 0, 12, 0, 120000)
        _check(torch_cuda, 64, hobjs, recs)
        hobjs = W.host_objects(G.CFG1, 0, 1)
        recs = G.records_host(G.CFG1, 0, 1, 0, 1 << 20)
        _check(torch_cuda, 16, hobjs, recs)
    finally:
        if old is None:
            del os.environ["VE_DENSE_BUDGET"]
        else:
            os.environ["VE_DENSE_BUDGET"] = old


@pytest.mark.parametrize("always", ["1", None])
def test_dense_gate_parity(torch_cuda, always):
    """The dense counters are used only by calls with >= 1 record per pre-snapshot element
    (VE_DENSE_ALWAYS=1 forces them): a chunked trace then mixes dense-counted and hash-counted
    calls for the same keys.  Results must not depend on which path counted what."""
    import os
    old = os.environ.get("VE_DENSE_ALWAYS")
    if always:
        os.environ["VE_DENSE_ALWAYS"] = always
    try:
        hobjs = W.host_objects(G.FUZZ, 0, 13)
        recs = G.records_host(G.FUZZ, 0, 13, 0, 150000)
        _check(torch_cuda, 64, hobjs, recs, chunks=[7, 40000, 41000, 100000])
        hobjs = W.host_objects(G.CFG1, 0, 1)
        recs = G.records_host(G.CFG1, 0, 1, 0, 1 << 20)
        _check(torch_cuda, 16, hobjs, recs, chunks=[5000, 1 << 19, (1 << 19) + 3])
    finally:
        if old is None:
            os.environ.pop("VE_DENSE_ALWAYS", None)
        else:
            os.environ["VE_DENSE_ALWAYS"] = old


def test_diff_before_report(torch_cuda):
    """ve_snapshot_diff before ve_report (the bench order): n_untouched must already count the
    elements of loads that are counted densely (their L bits are set when the counts are flushed)."""
    ve = _ve()
    for cfgc, seed, n, npcs in ((G.FUZZ, 7, 100000, 64), (G.CFG1, 1, 1 << 20, 16)):
        hobjs = W.host_objects(cfgc, 0, seed)
        recs = G.records_host(cfgc, 0, seed, 0, n)
        ctx = ve.Context(n_pcs=npcs, max_objects=max(len(hobjs), 1), hist_capacity=1 << 20)
        ctx.set_objects(W.device_objects(hobjs))
        ctx.analyze_records(W.device_records(recs), n)
        cfg = O.make_config(npcs)
        for o in hobjs:
            if o.get("pre") is None or o.get("post") is None:
                continue
            gd = ctx.snapshot_diff(o["id"], O.DIFF_WRITTEN)
            od = O.snapshot_diff(cfg, hobjs, recs, o["id"], O.DIFF_WRITTEN)
            assert not parity.compare_diff(gd, od), (cfgc, o["id"])
        okeys, oglob, oobj = O.analyze(cfg, hobjs, recs)
        assert not parity.compare_with_oracle(ctx.report(), okeys, oglob, oobj)
        ctx.close()


def test_analyze_records_host_parity(torch_cuda):
    """ve_analyze_records_host: host records streamed through the two staging buffers (2 Mi records
    each, copies on a side stream overlapped with the analysis) -- several chunks, a ragged tail."""
    ve = _ve()
    seed, n = 13, (1 << 21) * 2 + 12345
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    recs = G.records_host(G.FUZZ, 0, seed, 0, n)
    cfg = O.make_config(64)
    okeys, oglob, oobj = O.analyze(cfg, hobjs, recs)
    import torch
    ctx = ve.Context(n_pcs=64, max_objects=8, hist_capacity=1 << 22)
    ctx.set_objects(W.device_objects(hobjs))
    pinned = torch.from_numpy(recs.view(np.uint8)).pin_memory()
    ctx.analyze_records_host(pinned, n)
    assert not parity.compare_with_oracle(ctx.report(), okeys, oglob, oobj)
    ctx.reset()
    ctx.set_objects(W.device_objects(hobjs))
    ctx.analyze_records_host(recs, n)                 # pageable numpy memory
    assert not parity.compare_with_oracle(ctx.report(), okeys, oglob, oobj)
    ctx.close()
