"""S13 dump parity (SURVEY 4 "full report from GPU == oracle (binary dump
memcmp)"): the file ve_report_dump writes equals, byte for byte, the dump
include/ve.h specifies built from the CPU oracle's report (tests/dump_spec.py);
the JSON dump parses to the same object."""
import json
import os

import pytest

from gen import vegen as G
from oracle import oracle as O
from tests import dump_spec as D, workloads as W

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def _dumps(tmp_path, n_pcs, hobjs, recs, topk):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    ctx = ve.Context(n_pcs=n_pcs, max_objects=max(len(hobjs), 1), topk=topk, hist_capacity=1 << 20)
    ctx.set_objects(W.device_objects(hobjs))
    ctx.analyze_records(W.device_records(recs), len(recs))
    rep = ctx.report()
    pb, pj = os.path.join(tmp_path, "r.bin"), os.path.join(tmp_path, "r.json")
    rep.dump(pb, 0)
    rep.dump(pj, 1)
    rep.close()
    ctx.close()
    with open(pb, "rb") as f:
        gb = f.read()
    with open(pj) as f:
        gj = json.load(f)
    return gb, gj


@pytest.mark.parametrize("case", ["cfg1", "fuzz", "fuzz_top3"])
def test_dump_matches_oracle(torch_cuda, tmp_path, case):
    if case == "cfg1":
        n_pcs, topk = 16, 8
        hobjs = W.host_objects(G.CFG1, 0, 1)
        recs = G.records_host(G.CFG1, 0, 1, 0, 1 << 20)
    else:
        n_pcs, topk = 64, (3 if case == "fuzz_top3" else 8)
        hobjs = W.host_objects(G.FUZZ, 0, 11)
        recs = G.records_host(G.FUZZ, 0, 11, 0, 200003)
    okeys, oglob, oobj = O.analyze(O.make_config(n_pcs, topk=topk), hobjs, recs)
    gb, gj = _dumps(str(tmp_path), n_pcs, hobjs, recs, topk)
    want = D.oracle_dump_bytes(okeys, oglob, oobj, topk)
    got = D.mask_hist_entries(gb)
    assert got == want, D.first_difference(got, want, len(okeys), topk)
    wj = D.oracle_dump_json(okeys, oglob, oobj)
    assert gj == wj, next((f"key {a['key']}" for a, b in zip(gj["keys"], wj["keys"]) if a != b), "globals/objects")
