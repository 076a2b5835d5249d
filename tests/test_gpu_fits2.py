"""GPU parity of the f2 fit variants with the oracle, every field of every key bit-exact:
ve_dyadic_fit_ex(VE_FIT_TRUNC) against C22 (approximate structured) and ve_outlier_fit against C23
(structured with <= eps outliers), plain and truncated, on the hand-built role set of
tests/test_oracle_dyadic.py, srad_v1-style clamped ramps, and the cfg1 / cfg3 / cfg4 / cfg5 / fuzz
workloads."""
import numpy as np
import pytest

from gen import vegen as G
from oracle import oracle as O
from tests import test_oracle_dyadic as TD, workloads as W

pytestmark = pytest.mark.gpu

DY = ("state", "scale", "px", "qx", "py", "qy")
OF = ("state", "scale", "ax", "bx", "ay", "by", "n_off", "n")


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def _ctx(n_pcs, hobjs):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    ctx = ve.Context(n_pcs=n_pcs, max_objects=max(len(hobjs), 1), hist_capacity=1 << 20)
    ctx.set_objects(W.device_objects(hobjs))
    return ctx


def _compare(got, want, fields):
    assert len(got) == len(want)
    bad = []
    for f in fields:
        for k in np.nonzero(got[f].astype(np.int64) != want[f].astype(np.int64))[0][:20]:
            bad.append(f"key {k} {f}: gpu {got[f][k]} oracle {want[f][k]}")
    assert not bad, "\n".join(bad)


def _all(n_pcs, hobjs, recs):
    cfg = O.make_config(n_pcs)
    ctx = _ctx(n_pcs, hobjs)
    d = W.device_records(recs)
    n = len(recs)
    _compare(ctx.dyadic_fit_trunc(d, n), O.dyadic_fit_trunc(cfg, hobjs, recs), DY)
    _compare(ctx.outlier_fit(d, n), O.outlier_fit(cfg, hobjs, recs), OF)
    _compare(ctx.outlier_fit(d, n, flags=1), O.outlier_fit(cfg, hobjs, recs, flags=1), OF)
    ctx.close()


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_fits2_roles(torch_cuda, seed):
    rng = np.random.default_rng(seed)
    rs = TD.roles(rng)
    rows = [(int(x), int(b), pc, m) for pc, (_, pts, m) in enumerate(rs) for x, b in pts]
    rows = [rows[i] for i in rng.permutation(len(rows))]
    rows += [(x, b, pc, m | 0x20) for (x, b, pc, m) in rows[:10]]
    recs = np.array(rows, dtype=TD.REC)
    objs = [{"base": TD.BASE, "size": 24, "id": 0, "elem_width": 4, "pre": None, "post": None}]
    _all(len(rs), objs, recs)


def test_fits2_srad_clamped(torch_cuda):
    """srad_v1-style i32 ramps with clamped boundaries, several PCs, many warps"""
    N = 100003
    rows = []
    for pc, (lo_clamp, hi_clamp) in enumerate([(True, False), (False, True), (True, True), (False, False)]):
        for i in range(N):
            y = i - 1
            if lo_clamp and i == 0:
                y = 0
            if hi_clamp and i == N - 1:
                y = N - 3
            rows.append((TD.BASE + 0x100000 * pc + 4 * i, y & 0xFFFFFFFF, pc, TD.meta(2, 1)))
    recs = np.array(rows, dtype=TD.REC)
    objs = [{"base": TD.BASE, "size": 0x400000, "id": 0, "elem_width": 4, "pre": None, "post": None}]
    _all(4, objs, recs)
    o = O.outlier_fit(O.make_config(4), objs, recs)
    assert [int(o[p]["n_off"]) for p in range(4)] == [1, 1, 2, 0]


@pytest.mark.parametrize("cfg,epoch,seed", [(G.CFG1, 0, 1), (G.scaled(G.CFG4, 4), 0, 4), (G.scaled(G.CFG4, 4), 1, 4),
                                            (G.scaled(G.CFG3, 6), 0, 3), (G.scaled(G.CFG5, 0), 2024, 5)])
def test_fits2_workloads(torch_cuda, cfg, epoch, seed):
    inf = G.info(cfg, epoch)
    recs = G.records_host(cfg, epoch, seed, 0, inf["n_records"])
    _all(inf["n_pcs"], W.host_objects(cfg, epoch, seed), recs)


def test_fits2_fuzz(torch_cuda):
    inf = G.info(G.FUZZ, 0)
    recs = G.records_host(G.FUZZ, 0, 9, 0, 300_000)
    _all(inf["n_pcs"], W.host_objects(G.FUZZ, 0, 9), recs)
