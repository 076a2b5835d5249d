"""GPU: the full-size cfg5 duplicate scan (1000 objects, ~19.7 GiB of post snapshots)
against the closed form of the generator's duplicate classes (pinned to the oracle in
tests/test_oracle_cfg5.py), plus a scaled set against the oracle itself."""
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


def _device_set(torch, objs, seed, unit):
    s = torch.cuda.current_stream().cuda_stream
    out = []
    for o in objs:
        t = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
        G.dedup_device(seed, o["id"], unit, t.data_ptr(), s)
        out.append(dict(o, pre=None, post=t))
    torch.cuda.synchronize()
    return out


def test_cfg5_dedup_scaled_vs_oracle(torch_cuda):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    seed, n, unit = 5, 150, 8192
    objs = W.cfg5_dedup_objects(n, unit, seed)
    hobjs = [dict(o, pre=None, post=G.dedup_host(seed, o["id"], unit)) for o in objs]
    ctx = ve.Context(n_pcs=1, max_objects=1)
    g = ctx.object_dedup(_device_set(torch_cuda, objs, seed, unit))
    assert list(g) == list(O.object_dedup(hobjs))


def test_cfg5_dedup_full_size(torch_cuda):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    objs = W.cfg5_dedup_objects()
    assert sum(o["size"] for o in objs) > 19 << 30
    dobjs = _device_set(torch_cuda, objs, W.CFG5_SEED, W.CFG5_UNIT)
    ctx = ve.Context(n_pcs=1, max_objects=1)
    g = ctx.object_dedup(dobjs)
    assert list(g) == W.cfg5_expected_groups(objs)
    del dobjs
    torch_cuda.cuda.empty_cache()


# ---- cfg5 records half: kernels of the 4000-kernel application, one context reused across kernels --

from tests import cfg5k, parity  # noqa: E402


def _kernel_objects(torch, cfg, k, seed):
    s = torch.cuda.current_stream().cuda_stream
    out = []
    for i, o in enumerate(G.objects(cfg, k)):
        d = {f: o[f] for f in ("base", "size", "id", "elem_width")}
        for side in ("pre", "post"):
            t = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
            G.snapshot_device(cfg, k, seed, i, side == "post", t.data_ptr(), s)
            d[side] = t
        out.append(d)
    return out


def _largest_kernel():
    cfg = G.scaled(G.CFG5, 0)
    return max(range(4000), key=lambda k: G.info(cfg, k)["n_records"])


@pytest.mark.parametrize("shift,kernels", [(0, "sample"), (5, list(range(0, 4000, 211)))])
def test_cfg5_kernels_parity(torch_cuda, shift, kernels):
    """bit-exact against the oracle kernel by kernel, in bench.py's call order on ONE context with
    n_pcs = 64 (set_objects + analyze + report per kernel); full size on a sample that includes the
    largest kernel (1.68 M records), scaled on every 211th kernel"""
    from paper_conf_asplos_zhouhmm022_b200 import ve
    torch = torch_cuda
    cfg = G.scaled(G.CFG5, shift)
    if kernels == "sample":
        kernels = [_largest_kernel(), 0, 1, 7, 2024, 3999]
    seed = 5
    ocfg = O.make_config(64)
    ctx = ve.Context(n_pcs=64, max_objects=4, hist_capacity=1 << 23)
    s = torch.cuda.current_stream().cuda_stream
    bad = []
    for k in kernels:
        inf = G.info(cfg, k)
        n = inf["n_records"]
        dobjs = _kernel_objects(torch, cfg, k, seed)
        recs = torch.empty(n * 24, dtype=torch.uint8, device="cuda")
        G.records_device(cfg, k, seed, 0, n, recs.data_ptr(), s)
        ctx.set_objects(dobjs)
        ctx.analyze_records(recs, n, stream=s)
        rep = ctx.report()
        hrecs = G.records_host(cfg, k, seed, 0, n)
        okeys, oglob, oobj = O.analyze(ocfg, W.host_objects(cfg, k, seed), hrecs)
        bad += [f"kernel {k}: " + m for m in parity.compare_with_oracle(rep, okeys, oglob, oobj)]
        bad += cfg5k.check_cfg5_kernel({f: rep.keys[f] for f in rep.keys.dtype.names},
                                       rep.globals["n_records"], cfg, k)
    ctx.close()
    assert not bad, "\n".join(bad[:40])
