"""cfg5 duplicate-object scan: the closed form of the generator's duplicate
classes (tests/workloads.py) agrees with the oracle's C11 (pairwise memcmp) on scaled sets, so
the full-size GPU run can be checked against the closed form (test_gpu_cfg5.py, bench.py).
Records half: the 4000-kernel recipe and the oracle pinned by its closed forms (tests/cfg5k.py)."""
import numpy as np
import pytest

from gen import vegen as G
from oracle import oracle as O
from tests import workloads as W


@pytest.mark.parametrize("seed,n,unit", [(5, 120, 4096), (6, 200, 512), (5, 60, 64)])
def test_cfg5_closed_form_matches_oracle(seed, n, unit):
    objs = W.cfg5_dedup_objects(n, unit, seed)
    hobjs = [dict(o, pre=None, post=G.dedup_host(seed, o["id"], unit)) for o in objs]
    assert list(O.object_dedup(hobjs)) == W.cfg5_expected_groups(objs)


# ---- cfg5 records half: the 4000-kernel application (SURVEY 8(d) cfg5 "Kernels") ----------------

from tests import cfg5k  # noqa: E402


def test_cfg5_kernel_set_recipe():
    """4000 kernels, 4..64 PCs, 1..4 objects, exactly 10^9 records in total (groups of 8 sum to 2*10^6)."""
    cfg = G.scaled(G.CFG5, 0)
    infos = [G.info(cfg, k) for k in range(4000)]
    assert sum(i["n_records"] for i in infos) == 1_000_000_000
    for g in range(0, 4000, 8):
        assert sum(i["n_records"] for i in infos[g:g + 8]) == 2_000_000
    assert all(4 <= i["n_pcs"] <= 64 and 1 <= i["n_obj"] <= 4 for i in infos)
    assert {i["n_pcs"] for i in infos} == set(range(4, 65)) and {i["n_obj"] for i in infos} == {1, 2, 3, 4}
    with pytest.raises(ValueError):
        G.info(cfg, 4000)


@pytest.mark.parametrize("k", [0, 1, 7, 123, 2024, 3999])
def test_cfg5_kernel_layout(k):
    """every record lies in one object, each element is touched at most once, loads read pre,
    stores leave their value in post, untouched elements keep pre (post = pre + the stores)"""
    cfg = G.scaled(G.CFG5, 5)
    inf = G.info(cfg, k)
    recs = G.records_host(cfg, k, 5, 0, inf["n_records"])
    covered = 0
    for i, o in enumerate(G.objects(cfg, k)):
        m = (recs["addr"] >= o["base"]) & (recs["addr"] < o["base"] + o["size"])
        covered += int(m.sum())
        pre = G.snapshot_host(cfg, k, 5, i, 0).view(np.uint32)
        post = G.snapshot_host(cfg, k, 5, i, 1).view(np.uint32)
        e = (recs["addr"][m] - o["base"]) // 4
        st = ((recs["meta"][m] >> 4) & 1) == 1
        assert len(np.unique(e)) == len(e)
        assert np.array_equal(post[e[st]], recs["value"][m][st].astype(np.uint32))
        assert np.array_equal(pre[e[~st]], recs["value"][m][~st].astype(np.uint32))
        rest = np.setdiff1d(np.arange(len(pre)), e)
        assert np.array_equal(pre[rest], post[rest])
    assert covered == len(recs)


@pytest.mark.parametrize("shift,kernels", [(5, [0, 1, 7, 123, 500, 2024, 3999]), (0, [7, 9])])
def test_cfg5_oracle_closed_forms(shift, kernels):
    """the oracle's per-PC counts, redundant-store counts and single-value / single-zero flags on
    cfg5 kernels equal the recipe's closed forms (tests/cfg5k.py)"""
    cfg = G.scaled(G.CFG5, shift)
    for k in kernels:
        inf = G.info(cfg, k)
        recs = G.records_host(cfg, k, 5, 0, inf["n_records"])
        keys, glob, _ = O.analyze(O.make_config(inf["n_pcs"]), W.host_objects(cfg, k, 5), recs)
        bad = cfg5k.check_cfg5_kernel(keys, glob["n_records"], cfg, k)
        assert not bad, "\n".join(bad[:20])
