"""Pins of the CPU oracle on the cfg3 (PyTorch op mix) and cfg4 (f64 stencil)
workloads at reduced sizes: every closed form of tests/cfg34.py (derived from
the recipe), plus counts taken directly from the records."""
import numpy as np
import pytest

from gen import vegen as G
from oracle import oracle as O
from tests import cfg34, workloads as W


def _run(cfg, epoch, seed):
    inf = G.info(cfg, epoch)
    recs = G.records_host(cfg, epoch, seed, 0, inf["n_records"])
    hobjs = W.host_objects(cfg, epoch, seed)
    keys, glob, objs = O.analyze(O.make_config(inf["n_pcs"]), hobjs, recs)
    return recs, keys, glob, objs


@pytest.mark.parametrize("epoch", [0, 1])
def test_cfg4_closed_forms(epoch):
    shift = 4
    recs, keys, glob, objs = _run(G.scaled(G.CFG4, shift), epoch, 4)
    bad = cfg34.check_cfg4(keys, glob["n_records"], shift, epoch, objs)
    assert not bad, "\n".join(bad)
    if epoch == 0:
        v = recs["value"][recs["pc"] == 0]
        assert keys["n_distinct"][0] == len(np.unique(v))
        # T_in = 300 + 3q/8192 is an integer only for q = 0
        assert keys["n_nonint"][0] == int(np.count_nonzero(v != 0x4072C00000000000))


def test_cfg3_closed_forms():
    shift = 6
    recs, keys, glob, objs = _run(G.scaled(G.CFG3, shift), 0, 3)
    bad = cfg34.check_cfg3(keys, glob["n_records"], shift, objs)
    assert not bad, "\n".join(bad)
    # stores over a zero pre value are exactly the zero-valued stores of these PCs
    for pc in (2, 6, 8, 11):
        v = recs["value"][recs["pc"] == pc]
        assert keys["n_st_eq_pre"][pc] == int(np.count_nonzero(v == 0)), pc
    # the add output is the high-cardinality PC: its distinct values are the distinct sums
    assert keys["n_distinct"][6] == len(np.unique(recs["value"][recs["pc"] == 6]))
