"""GPU parity of every K1 (k_analyze) code path the bench runs, against the CPU oracle, bit-exact.

launch_analyze picks K1 v1 k_analyze<false> (single-key slots, run_dense) for traces with < 8 PCs
and K1 v2 k_analyze2 (register key slots, post-value counting) otherwise; VE_K1=1/2 and
VE_K1_MULTI=0/1 force one, so each trace below runs through v1 single-key, v1 multi-key and v2.  Traces of >= 4 x 148 x 16 x 16 windows (~4.85 M records)
take the 16-window static-interleave chunk path (multi-stage chunks), shorter ones one-stage chunks:
the large cases cover the chunk path the full-size configs use.

Inputs: the seeded generator (FUZZ, cfg2's gemm epoch, cfg3 / cfg4 scaled), the FUZZ trace
re-labelled onto 5 PCs (an input transformation: pc mod 5, the invalid PCs 64..69 kept invalid as
5..10), so the few-PC kernel sees chaos lanes, mixed types and more keys than its 4 slots.
"""
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


from tests.gpu_run import _check, _run_gpu  # noqa: E402


KERNELS = [("1", "0"), ("1", "1"), ("2", "")]     # (VE_K1, VE_K1_MULTI): v1 single-key, v1 multi-key, v2


class _k1:
    """force one k_analyze kernel for the block"""

    def __init__(self, k):
        self.k = k

    def __enter__(self):
        self.old = (os.environ.get("VE_K1"), os.environ.get("VE_K1_MULTI"))
        os.environ["VE_K1"], os.environ["VE_K1_MULTI"] = self.k
        return self

    def __exit__(self, *a):
        for name, v in zip(("VE_K1", "VE_K1_MULTI"), self.old):
            if v is None:
                os.environ.pop(name, None)
            else:
                os.environ[name] = v


def fuzz5(seed, n, r0=0):
    """FUZZ records re-labelled onto 5 PCs (input transformation only)."""
    recs = G.records_host(G.FUZZ, 0, seed, r0, n)
    pc = recs["pc"].astype(np.int64)
    recs["pc"] = np.where(pc < 64, pc % 5, 5 + (pc - 64)).astype(np.uint32)
    return recs


def _parity(torch_cuda, n_pcs, hobjs, recs, hcap=1 << 22, chunks=None):
    cfg = O.make_config(n_pcs)
    okeys, oglob, oobj = O.analyze(cfg, hobjs, recs)
    for k in KERNELS:
        with _k1(k):
            rep, _ = _run_gpu(torch_cuda, n_pcs, hobjs, recs, hist_capacity=hcap, chunks=chunks)
        bad = parity.compare_with_oracle(rep, okeys, oglob, oobj)
        assert not bad, f"kernel {k}:\n" + "\n".join(bad[:30])


@pytest.mark.parametrize("seed,n", [(21, 4096), (22, 100003), (23, 300001), (24, 1 << 20)])
def test_fuzz5_both_kernels(torch_cuda, seed, n):
    """few-PC FUZZ: the single-key kernel (the cfg2 headline's) on adversarial windows"""
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    recs = fuzz5(seed, n)
    _check(torch_cuda, 5, hobjs, recs)           # default selection (< 8 PCs: k_analyze<false>), with the diffs
    _parity(torch_cuda, 5, hobjs, recs)


def test_fuzz5_chunked_both_kernels(torch_cuda):
    seed, n = 25, 400009
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    _parity(torch_cuda, 5, hobjs, fuzz5(seed, n), chunks=[31, 100000, 100001, 250000])


def test_cfg1_both_kernels(torch_cuda):
    hobjs = W.host_objects(G.CFG1, 0, 1)
    _parity(torch_cuda, 16, hobjs, G.records_host(G.CFG1, 0, 1, 0, 1 << 20))


@pytest.mark.slow
@pytest.mark.parametrize("which", ["fuzz64", "fuzz5"])
def test_fuzz_chunk_path_8m(torch_cuda, which):
    """8.4 M records (> 4.85 M): the 16-window static-interleave chunk path, both kernels"""
    seed, n = 26, 8_400_017
    hobjs = W.host_objects(G.FUZZ, 0, seed)
    if which == "fuzz5":
        _parity(torch_cuda, 5, hobjs, fuzz5(seed, n), hcap=1 << 23)
    else:
        _parity(torch_cuda, 64, hobjs, G.records_host(G.FUZZ, 0, seed, 0, n), hcap=1 << 23)


@pytest.mark.slow
def test_cfg2_gemm_16m_sample(torch_cuda):
    """The cfg2 gemm epoch's first 16 M records (A / B / C interleaved as in the full trace, 5 PCs),
    full snapshots: the bench's oracle sample, now compared field by field on both kernels."""
    seed = G.SEEDS[G.CFG2]
    n = 16_000_000
    hobjs = W.host_objects(G.CFG2, 1, seed)
    recs = G.records_host(G.CFG2, 1, seed, 0, n)
    _parity(torch_cuda, G.info(G.CFG2, 1)["n_pcs"], hobjs, recs)


@pytest.mark.slow
def test_cfg2_gemm_16m_offset_sample(torch_cuda):
    """16 M gemm records from the middle of the epoch (another tile mix, ragged start)"""
    seed = G.SEEDS[G.CFG2]
    n, r0 = 16_000_003, 100_000_013
    hobjs = W.host_objects(G.CFG2, 1, seed)
    recs = G.records_host(G.CFG2, 1, seed, r0, n)
    _parity(torch_cuda, G.info(G.CFG2, 1)["n_pcs"], hobjs, recs)


@pytest.mark.slow
@pytest.mark.parametrize("epoch", [0, 1])
def test_cfg4_scaled_chunk_path(torch_cuda, epoch):
    """cfg4 at 1/8 of the grid per axis (shift 3: 64^3 points, 2.1 / 1.8 M records) and shift 2
    (128^3: 16.8 / 14.7 M records, the chunk path) -- both kernels"""
    for shift in (3, 2):
        cfg = G.scaled(G.CFG4, shift)
        inf = G.info(cfg, epoch)
        hobjs = W.host_objects(cfg, epoch, 4)
        recs = G.records_host(cfg, epoch, 4, 0, inf["n_records"])
        _parity(torch_cuda, inf["n_pcs"], hobjs, recs, hcap=1 << 22)


@pytest.mark.slow
def test_cfg3_scaled_chunk_path(torch_cuda):
    """cfg3 at shift 5 (8.3 M records, 20 PCs, 16 objects) -- both kernels"""
    cfg = G.scaled(G.CFG3, 5)
    inf = G.info(cfg, 0)
    hobjs = W.host_objects(cfg, 0, 3)
    recs = G.records_host(cfg, 0, 3, 0, inf["n_records"])
    _parity(torch_cuda, inf["n_pcs"], hobjs, recs, hcap=1 << 23)


def test_generator_device_equals_host(torch_cuda):
    """G0: the device generator writes exactly the host generator's bytes (records and snapshots), so
    the full-size runs that feed device-generated traces analyze the traces the oracle sees."""
    import torch
    cases = [(G.CFG1, 0, 1, [(0, 1 << 20)]),
             (G.CFG2, 0, 2, [(0, 100000), (5_914_600, 24)]),
             (G.CFG2, 1, 2, [(0, 300000), (123_456_789, 100001), (225_640_448 - 77, 77)]),
             (G.scaled(G.CFG3, 0), 0, 3, [(0, 200000), (700_000_000, 99999), (264_291_072 - 1000, 1000)]),
             (G.scaled(G.CFG4, 0), 0, 4, [(0, 200000), (999_999_999, 4096)]),
             (G.scaled(G.CFG4, 0), 1, 4, [(0, 200000), (939_524_096 - 513, 513)]),
             (G.FUZZ, 0, 7, [(0, 300001)])]
    sp = torch.cuda.current_stream().cuda_stream
    for cfg, ep, seed, ranges in cases:
        for r0, n in ranges:
            d = torch.empty(n * 24, dtype=torch.uint8, device="cuda")
            G.records_device(cfg, ep, seed, r0, n, d.data_ptr(), sp)
            h = G.records_host(cfg, ep, seed, r0, n)
            assert d.cpu().numpy().tobytes() == h.tobytes(), (cfg, ep, r0, n)
        for i, o in enumerate(G.objects(cfg, ep)):
            if o["size"] > (64 << 20):
                continue                          # host generation of 1 GiB fields is slow; their prefix below
            for post in (0, 1):
                d = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
                G.snapshot_device(cfg, ep, seed, i, post, d.data_ptr(), sp)
                assert d.cpu().numpy().tobytes() == G.snapshot_host(cfg, ep, seed, i, post).tobytes(), (cfg, ep, i)
        for i, o in enumerate(G.objects(cfg, ep)):
            if o["size"] <= (64 << 20):
                continue
            d = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
            G.snapshot_device(cfg, ep, seed, i, 1, d.data_ptr(), sp)
            for off in (0, o["size"] // 2 + 8, o["size"] - 4096):
                h = G.snapshot_host(cfg, ep, seed, i, 1, off, 4096)
                assert d[off:off + 4096].cpu().numpy().tobytes() == h.tobytes(), (cfg, ep, i, off)
            del d
    # cfg5 kernels (the records half's per-kernel traces and snapshots)
    cfg5 = G.scaled(G.CFG5, 0)
    for k in (0, 1, 1234, 3999):
        n = G.info(cfg5, k)["n_records"]
        d = torch.empty(n * 24, dtype=torch.uint8, device="cuda")
        G.records_device(cfg5, k, 5, 0, n, d.data_ptr(), sp)
        assert d.cpu().numpy().tobytes() == G.records_host(cfg5, k, 5, 0, n).tobytes(), k
        for i, o in enumerate(G.objects(cfg5, k)):
            for post in (0, 1):
                t = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
                G.snapshot_device(cfg5, k, 5, i, post, t.data_ptr(), sp)
                assert t.cpu().numpy().tobytes() == G.snapshot_host(cfg5, k, 5, i, post).tobytes(), (k, i)
