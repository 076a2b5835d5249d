"""cfg5 duplicate-object scan: the closed form of the generator's duplicate
classes (tests/workloads.py) agrees with the oracle's C11 (pairwise memcmp) on scaled sets, so
the full-size GPU run can be checked against the closed form (test_gpu_cfg5.py, bench.py)."""
import pytest

from gen import vegen as G
from oracle import oracle as O
from tests import workloads as W


@pytest.mark.parametrize("seed,n,unit", [(5, 120, 4096), (6, 200, 512), (5, 60, 64)])
def test_cfg5_closed_form_matches_oracle(seed, n, unit):
    objs = W.cfg5_dedup_objects(n, unit, seed)
    hobjs = [dict(o, pre=None, post=G.dedup_host(seed, o["id"], unit)) for o in objs]
    assert list(O.object_dedup(hobjs)) == W.cfg5_expected_groups(objs)
