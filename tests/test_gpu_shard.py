"""GPU parity of the object-sharded S10 / S11: ve_snapshot_diff_all and
ve_object_dedup over G ranks, against the CPU oracle.

Transports: G same-device contexts playing ranks 0..G-1 (ve_*_group: device copies instead of
NCCL, the algorithm the NCCL path runs), a real 1-rank NCCL communicator, and -- when the box has
two GPUs -- two NCCL ranks in two processes.  Every rank must end with the oracle's full result."""
import os

import numpy as np
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


def _ve():
    from paper_conf_asplos_zhouhmm022_b200 import ve
    return ve


def _diff_expect(cfg, hobjs, recs, mode):
    out = {}
    for o in hobjs:
        if o.get("pre") is not None and o.get("post") is not None:
            out[o["id"]] = O.snapshot_diff(cfg, hobjs, recs, o["id"], mode)
    return out


def _check_diffs(got, want):
    bad = []
    for oid, od in want.items():
        bad += [f"obj {oid} " + b for b in parity.compare_diff(got[oid], od)]
    return bad


def _dedup_set(seed, n=48, unit=4096):
    objs = [G.dedup_object(seed, i, unit) for i in range(n)]
    host = [dict(o, pre=None, post=G.dedup_host(seed, i, unit)) for i, o in enumerate(objs)]
    host[5] = dict(host[5], post=None)                      # a NULL post: a singleton
    return host


@pytest.mark.parametrize("Gr", [2, 3])
def test_sharded_diff_and_dedup_group(torch_cuda, Gr):
    ve = _ve()
    seed, n = 31, 150001
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    recs = G.records_host(G.FUZZ, 0, seed, 0, n)
    cfg = O.make_config(64)
    dobjs = W.device_objects(hobjs)
    drec = W.device_records(recs)
    ctxs = []
    for r in range(Gr):
        lo, hi = ve.rank_chunk(n, r, Gr)
        c = ve.Context(n_pcs=64, max_objects=8, hist_capacity=1 << 20)
        c.set_objects(dobjs)
        c.analyze_records(drec[lo * 24:hi * 24], hi - lo)
        ctxs.append(c)
    ve.merge_group(ctxs)
    for mode in (O.DIFF_WRITTEN, O.DIFF_ALL):
        got = ve.snapshot_diff_all_group(ctxs, mode)
        bad = _check_diffs(got, _diff_expect(cfg, hobjs, recs, mode))
        assert not bad, "\n".join(bad[:20])
    # the duplicate scan over a set with zero objects, exact copies and one-bit flips
    hset = _dedup_set(7)
    want = O.object_dedup(hset)
    dset = [dict(o, post=torch_cuda.from_numpy(o["post"]).cuda() if o["post"] is not None else None) for o in hset]
    got = ve.object_dedup_group(ctxs, dset)
    assert list(got) == list(want)
    assert len(set(int(x) for x in want)) < len(want)        # duplicates exist


def test_diff_all_local_and_nccl_one_rank(torch_cuda):
    ve = _ve()
    seed, n = 32, 120007
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    recs = G.records_host(G.FUZZ, 0, seed, 0, n)
    cfg = O.make_config(64)
    c = ve.Context(n_pcs=64, max_objects=8, hist_capacity=1 << 20)
    c.set_objects(W.device_objects(hobjs))
    c.analyze_records(W.device_records(recs), n)
    want = _diff_expect(cfg, hobjs, recs, O.DIFF_WRITTEN)
    assert not _check_diffs(c.snapshot_diff_all(O.DIFF_WRITTEN), want)
    comm = ve.nccl_comm_init(ve.nccl_unique_id(), 0, 1)
    assert not _check_diffs(c.snapshot_diff_all(O.DIFF_WRITTEN, comm=comm), want)
    hset = _dedup_set(8)
    dset = [dict(o, post=torch_cuda.from_numpy(o["post"]).cuda() if o["post"] is not None else None) for o in hset]
    assert list(c.object_dedup(dset, comm=comm)) == list(O.object_dedup(hset))


def _two_rank_worker(rank, port, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE="2")
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", device_id=torch.device("cuda", rank))
    ve = _ve()
    seed, n = 33, 100003
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    recs = G.records_host(G.FUZZ, 0, seed, 0, n)
    comm = ve.nccl_comm_from_torch(rank, 2)
    lo, hi = ve.rank_chunk(n, rank, 2)
    c = ve.Context(n_pcs=64, max_objects=8, hist_capacity=1 << 20, device=rank)
    c.set_objects(W.device_objects(hobjs, device=f"cuda:{rank}"))
    c.analyze_records(W.device_records(recs[lo:hi], device=f"cuda:{rank}"), hi - lo)
    c.merge(comm=comm)
    rep = c.report()
    cfg = O.make_config(64)
    okeys, oglob, oobj = O.analyze(cfg, hobjs, recs)
    bad = parity.compare_with_oracle(rep, okeys, oglob, oobj)
    bad += _check_diffs(c.snapshot_diff_all(O.DIFF_WRITTEN, comm=comm), _diff_expect(cfg, hobjs, recs, O.DIFF_WRITTEN))
    hset = _dedup_set(9)
    dset = [dict(o, post=torch.from_numpy(o["post"]).cuda(rank) if o["post"] is not None else None) for o in hset]
    if list(c.object_dedup(dset, comm=comm)) != list(O.object_dedup(hset)):
        bad.append("dedup groups differ")
    q.put((rank, bad[:10]))
    dist.destroy_process_group()


def test_two_rank_nccl(torch_cuda):
    """S12 merge + sharded S10 / S11 over two NCCL ranks (two processes, one GPU each)"""
    if torch_cuda.cuda.device_count() < 2:
        pytest.skip("needs two GPUs (gpurun boxes give one; covered by the same-device group test above)")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29600 + os.getpid() % 1000
    ps = [ctx.Process(target=_two_rank_worker, args=(r, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=600) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    for rank, bad in res:
        assert not bad, f"rank {rank}: {bad}"
