"""GPU parity of SURVEY 8(f) f1 (PAPER.md 6.1): ve_interval_merge,
ve_record_intervals and ve_plan_copies against the oracle's C13-C15, bit-exact,
through the C ABI.  Sizes span many tiles (2048 intervals each) and ragged tails;
address spans force 1..6 radix passes; the sorted-input path skips the sort."""
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


def _ve():
    from paper_conf_asplos_zhouhmm022_b200 import ve
    return ve


def _gpu_merge(torch, ctx, iv):
    ve = _ve()
    n = len(iv)
    d_in = torch.from_numpy(np.ascontiguousarray(iv).view(np.uint8).copy()).cuda()
    d_out = torch.zeros(max(n, 1) * 16, dtype=torch.uint8, device="cuda")
    k = ctx.interval_merge(d_in, n, d_out)
    return d_out[:k * 16].cpu().numpy().view(ve.INTERVAL_DTYPE), d_out


def _random_intervals(seed, n, span_bits, max_len, empty_frac=0.05):
    rng = np.random.default_rng(seed)
    base = 0x7f0000000000 if span_bits < 47 else 0
    s = base + rng.integers(0, 1 << span_bits, n, dtype=np.uint64)
    ln = rng.integers(0, max_len, n, dtype=np.uint64)
    e = s + ln
    emp = rng.random(n) < empty_frac
    e[emp] = s[emp] - np.uint64(1)                   # start > end: empty
    iv = np.zeros(n, dtype=O.INTERVAL_DTYPE)
    iv["start"], iv["end"] = s, e
    return iv


@pytest.mark.parametrize("seed,n,span_bits,max_len", [
    (1, 1, 10, 4), (2, 31, 10, 4), (3, 2049, 12, 8), (4, 100003, 20, 64), (5, 250001, 47, 1 << 20),
    (6, 65536, 8, 3), (7, 300000, 30, 4096)])
def test_interval_merge_parity(torch_cuda, seed, n, span_bits, max_len):
    ve = _ve()
    ctx = ve.Context(n_pcs=1, max_objects=1)
    iv = _random_intervals(seed, n, span_bits, max_len)
    got, _ = _gpu_merge(torch_cuda, ctx, iv)
    want = O.interval_merge(iv)
    assert len(got) == len(want)
    assert np.array_equal(got["start"], want["start"]) and np.array_equal(got["end"], want["end"])
    ctx.close()


def test_interval_merge_edges(torch_cuda):
    ve = _ve()
    ctx = ve.Context(n_pcs=1, max_objects=1)
    top = (1 << 64) - 1
    cases = [
        [(5, 4)],                                             # only empty
        [(0, top), (7, 8)],                                   # everything
        [(top - 3, top), (5, 9), (top, top)],
        [(i, i) for i in range(5000)],                        # one adjacent chain over tiles (sorted: no sort pass)
        [(2 * i, 2 * i) for i in range(5000)][::-1],          # 1-byte gaps, reversed
        [(10, 20)] * 4097,                                    # duplicates across tiles
    ]
    for pairs in cases:
        iv = np.array(pairs, dtype=np.uint64).view(O.INTERVAL_DTYPE).ravel()
        got, _ = _gpu_merge(torch_cuda, ctx, iv)
        want = O.interval_merge(iv)
        assert got.tobytes() == want.tobytes(), pairs[:3]
    assert ctx.interval_merge(None, 0, None) == 0
    ctx.close()


@pytest.mark.parametrize("seed,n", [(1, 4096), (3, 100003)])
def test_record_intervals_fuzz_parity(torch_cuda, seed, n):
    ve = _ve()
    recs = G.records_host(G.FUZZ, 0, seed, 0, n)
    ctx = ve.Context(n_pcs=64, max_objects=8)
    d = W.device_records(recs)
    out = torch_cuda.zeros(n * 16, dtype=torch_cuda.uint8, device="cuda")
    k = ctx.record_intervals(d, n, out)
    got = out[:k * 16].cpu().numpy().view(ve.INTERVAL_DTYPE)
    want = O.record_intervals(64, recs)
    assert got.tobytes() == want.tobytes()
    # the copy plan over the fuzz objects
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    ctx.set_objects(W.device_objects(hobjs))
    for seg_max, dense in ((32, 50), (2, 10), (1 << 30, 100)):
        gp = ctx.plan_copies(out, k, seg_max, dense)
        op = O.plan_copies(hobjs, want, seg_max, dense)
        assert gp.tobytes() == op.tobytes()
    ctx.close()


def test_record_intervals_cfg1_and_plan(torch_cuda):
    ve = _ve()
    recs = G.records_host(G.CFG1, 0, 1, 0, 1 << 20)
    hobjs = W.host_objects(G.CFG1, 0, 1)
    ctx = ve.Context(n_pcs=16, max_objects=1)
    ctx.set_objects(W.device_objects(hobjs))
    d = W.device_records(recs)
    out = torch_cuda.zeros(len(recs) * 16, dtype=torch_cuda.uint8, device="cuda")
    k = ctx.record_intervals(d, len(recs), out)
    got = out[:k * 16].cpu().numpy().view(ve.INTERVAL_DTYPE)
    o = hobjs[0]
    assert k == 1 and int(got[0]["start"]) == o["base"] and int(got[0]["end"]) == o["base"] + o["size"] - 1
    plan = ctx.plan_copies(out, k)
    assert plan[0]["choice"] == ve.COPY_MINMAX and int(plan[0]["accessed_bytes"]) == o["size"]
    # a merged set that is not sorted / disjoint is rejected
    bad = torch_cuda.from_numpy(np.array([[10, 20], [15, 30]], dtype=np.uint64).view(np.uint8).ravel()).cuda()
    with pytest.raises(ve.VeError):
        ctx.plan_copies(bad, 2)
    ctx.close()


def test_record_intervals_cfg2_full_size(torch_cuda):
    """Full BASELINE configs[1] gemm epoch (225.6 M records): A, B and C cover the weights, workspace and
    output objects completely, and the objects are not adjacent -> exactly their three ranges (closed form)."""
    ve = _ve()
    torch = torch_cuda
    inf = G.info(G.CFG2, 1)
    n = inf["n_records"]
    recs = torch.empty(n * 24, dtype=torch.uint8, device="cuda")
    G.records_device(G.CFG2, 1, G.SEEDS[G.CFG2], 0, n, recs.data_ptr(), torch.cuda.current_stream().cuda_stream)
    out = torch.empty(4 * 16, dtype=torch.uint8, device="cuda")   # room for the merged set only
    big = torch.empty(n * 16, dtype=torch.uint8, device="cuda")
    ctx = ve.Context(n_pcs=inf["n_pcs"], max_objects=8)
    k = ctx.record_intervals(recs, n, big)
    got = big[:k * 16].cpu().numpy().view(ve.INTERVAL_DTYPE)
    objs = G.objects(G.CFG2, 1)[:3]
    assert k == 3
    for g, o in zip(got, objs):
        assert (int(g["start"]), int(g["end"])) == (o["base"], o["base"] + o["size"] - 1)
    del out
    ctx.close()
