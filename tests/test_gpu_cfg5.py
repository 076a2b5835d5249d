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
