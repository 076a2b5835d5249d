"""GPU parity of ve_dyadic_fit (f2: dyadic-scaled exact linear fit) with the oracle's C21, every
field of every key bit-exact: the hand-built role set of tests/test_oracle_dyadic.py (lines, one-ulp
misses, overflow of the 2^62 bound, NaN / inf, points, f16 / bf16 / f64 ramps, huge integers),
objects and the SHARED key, and the cfg1 / cfg3 / cfg4 / cfg5 / fuzz workloads (cfg4's f64 stencils
are where non-integral structured values live)."""
import numpy as np
import pytest

from gen import vegen as G
from oracle import oracle as O
from tests import test_oracle_dyadic as TD, workloads as W

pytestmark = pytest.mark.gpu

FIELDS = ("state", "scale", "px", "qx", "py", "qy")


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def _gpu(torch, n_pcs, hobjs, recs):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    ctx = ve.Context(n_pcs=n_pcs, max_objects=max(len(hobjs), 1), hist_capacity=1 << 20)
    ctx.set_objects(W.device_objects(hobjs))
    d = W.device_records(recs)
    out = ctx.dyadic_fit(d, len(recs))
    ctx.close()
    return out


def _compare(got, want):
    assert len(got) == len(want)
    bad = []
    for f in FIELDS:
        for k in np.nonzero(got[f].astype(np.int64) != want[f].astype(np.int64))[0][:20]:
            bad.append(f"key {k} {f}: gpu {got[f][k]} oracle {want[f][k]}")
    assert not bad, "\n".join(bad)


@pytest.mark.parametrize("seed", [0, 1])
def test_dyadic_roles(torch_cuda, seed):
    rng = np.random.default_rng(seed)
    rs = TD.roles(rng)
    rows = [(int(x), int(b), pc, m) for pc, (_, pts, m) in enumerate(rs) for x, b in pts]
    rows = [rows[i] for i in rng.permutation(len(rows))]
    # plus shared-space copies of the first roles and an object covering half of the addresses
    rows += [(x, b, pc, m | 0x20) for (x, b, pc, m) in rows[:10]]
    recs = np.array(rows, dtype=TD.REC)
    objs = [{"base": TD.BASE, "size": 24, "id": 0, "elem_width": 4, "pre": None, "post": None}]
    cfg = O.make_config(len(rs))
    want = O.dyadic_fit(cfg, objs, recs)
    _compare(_gpu(torch_cuda, len(rs), objs, recs), want)
    assert int(want[[n for n, _, _ in rs].index("f32 ramp")]["state"]) == 2


@pytest.mark.parametrize("cfg,epoch,seed", [(G.CFG1, 0, 1), (G.scaled(G.CFG4, 4), 0, 4), (G.scaled(G.CFG4, 4), 1, 4),
                                            (G.scaled(G.CFG3, 6), 0, 3), (G.scaled(G.CFG5, 0), 2024, 5)])
def test_dyadic_workloads(torch_cuda, cfg, epoch, seed):
    inf = G.info(cfg, epoch)
    recs = G.records_host(cfg, epoch, seed, 0, inf["n_records"])
    hobjs = W.host_objects(cfg, epoch, seed)
    want = O.dyadic_fit(O.make_config(inf["n_pcs"]), hobjs, recs)
    _compare(_gpu(torch_cuda, inf["n_pcs"], hobjs, recs), want)


def test_dyadic_fuzz(torch_cuda):
    inf = G.info(G.FUZZ, 0)
    recs = G.records_host(G.FUZZ, 0, 9, 0, 300_000)
    hobjs = W.host_objects(G.FUZZ, 0, 9)
    want = O.dyadic_fit(O.make_config(inf["n_pcs"]), hobjs, recs)
    _compare(_gpu(torch_cuda, inf["n_pcs"], hobjs, recs), want)


def test_dyadic_empty(torch_cuda):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    ctx = ve.Context(n_pcs=3, max_objects=1, hist_capacity=1 << 16)
    ctx.set_objects([])
    got = ctx.dyadic_fit(None, 0)
    ctx.close()
    assert len(got) == 4 and (got["state"] == 0).all()
