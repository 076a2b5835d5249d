"""GPU parity on the cfg3 (PyTorch op mix) and cfg4 (f64 stencil) workloads:
bit-exact against the CPU oracle at reduced sizes (every field of the report),
and the recipe's closed forms (tests/cfg34.py) at FULL size -- 264 M records
(cfg3) and 1.07 G + 0.94 G records (cfg4), generated on the device in chunks
and analysed through repeated ve_analyze_records calls, as bench.py does."""
import numpy as np
import pytest

from gen import vegen as G
from oracle import oracle as O
from tests import cfg34, workloads as W
from tests.gpu_run import _check, _ve

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


@pytest.mark.parametrize("epoch", [0, 1])
def test_cfg4_parity_small(torch_cuda, epoch):
    cfg = G.scaled(G.CFG4, 4)
    inf = G.info(cfg, epoch)
    recs = G.records_host(cfg, epoch, 4, 0, inf["n_records"])
    _check(torch_cuda, inf["n_pcs"], W.host_objects(cfg, epoch, 4), recs, hist_capacity=1 << 20)


@pytest.mark.parametrize("epoch,seed", [(0, 3), (2, 5)])
def test_cfg3_parity_small(torch_cuda, epoch, seed):
    cfg = G.scaled(G.CFG3, 6)
    inf = G.info(cfg, epoch)
    recs = G.records_host(cfg, epoch, seed, 0, inf["n_records"])
    _check(torch_cuda, inf["n_pcs"], W.host_objects(cfg, epoch, seed), recs, hist_capacity=1 << 22)


def _full_report(torch, cfg, epoch, seed, hist_capacity, chunk=1 << 27):
    """Analyse a full-size epoch: snapshots and records generated on the device."""
    ve = _ve()
    inf = G.info(cfg, epoch)
    n = inf["n_records"]
    stream = torch.cuda.current_stream()
    dobjs = []
    for i, o in enumerate(G.objects(cfg, epoch)):
        d = {k: o[k] for k in ("base", "size", "id", "elem_width")}
        for side in ("pre", "post"):
            t = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
            G.snapshot_device(cfg, epoch, seed, i, side == "post", t.data_ptr(), stream.cuda_stream)
            d[side] = t
        dobjs.append(d)
    ctx = ve.Context(n_pcs=inf["n_pcs"], max_objects=len(dobjs), hist_capacity=hist_capacity)
    ctx.set_objects(dobjs)
    buf = torch.empty(min(chunk, n) * 24, dtype=torch.uint8, device="cuda")
    for r0 in range(0, n, chunk):
        m = min(chunk, n - r0)
        G.records_device(cfg, epoch, seed, r0, m, buf.data_ptr(), stream.cuda_stream)
        ctx.analyze_records(buf, m, stream=stream.cuda_stream)
    rep = ctx.report()
    k = {f: rep.keys[f] for f in rep.keys.dtype.names}
    k["top_bits"], k["top_count"] = rep.topk["bits"], rep.topk["count"]
    out = (k, int(rep.globals["n_records"]), rep.objects)
    ctx.close()
    del dobjs, buf
    torch.cuda.empty_cache()
    return out


@pytest.mark.parametrize("epoch", [0, 1])
def test_cfg4_full_size_closed_forms(torch_cuda, epoch):
    k, n, objs = _full_report(torch_cuda, G.scaled(G.CFG4, 0), epoch, 4, 1 << 22)
    bad = cfg34.check_cfg4(k, n, 0, epoch, objs)
    assert not bad, "\n".join(bad)


def test_cfg3_full_size_closed_forms(torch_cuda):
    k, n, objs = _full_report(torch_cuda, G.scaled(G.CFG3, 0), 0, 3, 1 << 25)
    bad = cfg34.check_cfg3(k, n, 0, objs)
    assert not bad, "\n".join(bad)
