"""ve_set_units / ve_analyze_units: several independent traces in one launch equal each trace
analysed alone by the oracle, its PCs shifted to the unit's pc_base and its objects' ids to the
unit's first id (C12; include/ve.h).  The FUZZ units reuse the same object addresses with
different snapshots, so a unit's addresses must map to its own objects only; FUZZ's invalid PCs
(64..69) must stay invalid, its shared-space records add into the one SHARED key."""
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


def _units(seeds_fuzz, cfg5_kernels):
    units = []
    for seed, n in seeds_fuzz:
        units.append(dict(npc=64, hobjs=W.host_objects(G.FUZZ, 0, seed), recs=G.records_host(G.FUZZ, 0, seed, 0, n)))
    cfg = G.scaled(G.CFG5, 0)
    for k in cfg5_kernels:
        inf = G.info(cfg, k)
        n = min(inf["n_records"], 300000)
        units.append(dict(npc=inf["n_pcs"], hobjs=W.host_objects(cfg, k, 5), recs=G.records_host(cfg, k, 5, 0, n)))
    return units


def _cmp_key(g, gi, o, oi, what):
    bad = []
    for f in parity.RAW_FIELDS + parity.DERIVED:
        if int(g[f][gi]) != int(o[f][oi]):
            bad.append(f"{what} {f}: gpu {g[f][gi]} oracle {o[f][oi]}")
    if not np.array_equal(g["n_type"][gi], o["n_type"][oi].astype(g["n_type"].dtype)):
        bad.append(f"{what} n_type")
    if int(o["line_state"][oi]) in (O.LINE_POINT, O.LINE_LINE):
        for f in parity.ENDPOINTS:
            if int(g[f][gi]) != int(o[f][oi]):
                bad.append(f"{what} {f}")
    return bad


@pytest.mark.parametrize("case", ["fuzz", "mixed"])
def test_units_match_oracle_per_unit(torch_cuda, case):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    torch = torch_cuda
    if case == "fuzz":
        units = _units([(41, 70001), (42, 4097), (43, 31), (44, 150003), (45, 0), (46, 64)], [])
    else:
        units = _units([(47, 50001)], [0, 7, 400, 1234])
    # device records: every unit at a 16-byte aligned offset (an even record index)
    offs, tot = [], 0
    for u in units:
        offs.append(tot)
        tot += len(u["recs"]) + (len(u["recs"]) & 1)
    buf = np.zeros(max(tot, 2), dtype=units[0]["recs"].dtype)
    for u, o in zip(units, offs):
        buf[o:o + len(u["recs"])] = u["recs"]
    drec = W.device_records(buf)
    pcb, obase, dunits, uobjs = 0, 0, [], []
    for u, o in zip(units, offs):
        u["pcb"], u["obase"] = pcb, obase
        dobjs = W.device_objects(u["hobjs"])
        for d in dobjs:
            d["id"] += obase
        uobjs.append(dobjs)
        dunits.append((drec.data_ptr() + o * 24, len(u["recs"]), pcb, u["npc"]))
        pcb += u["npc"]
        obase += len(u["hobjs"])
    n_pcs, n_obj = pcb, obase
    ctx = ve.Context(n_pcs=n_pcs, max_objects=n_obj, hist_capacity=1 << 21)
    for rep_i in range(2):                       # twice: the second epoch reuses the ctx
        ctx.set_units(uobjs)
        ctx.analyze_units(dunits)
        rep = ctx.report()
        bad = []
        shared = {"n_ld": 0, "n_st": 0, "n_zero": 0}
        glob = {"n_records": 0, "n_invalid": 0, "n_unmapped": 0}
        for i, u in enumerate(units):
            okeys, oglob, oobj = O.analyze(O.make_config(u["npc"]), u["hobjs"], u["recs"])
            for p in range(u["npc"]):
                bad += _cmp_key(rep.keys, u["pcb"] + p, okeys, p, f"unit {i} pc {p}")
                nt = int(okeys["n_top"][p])
                if not (np.array_equal(rep.topk["bits"][u["pcb"] + p, :nt], okeys["top_bits"][p, :nt]) and
                        np.array_equal(rep.topk["count"][u["pcb"] + p, :nt], okeys["top_count"][p, :nt])):
                    bad.append(f"unit {i} pc {p} topk")
            for j in range(len(u["hobjs"])):
                gk, ok = n_pcs + u["obase"] + j, u["npc"] + j
                bad += _cmp_key(rep.keys, gk, okeys, ok, f"unit {i} object {j}")
                for f in parity.OBJ_FIELDS:
                    if int(rep.objects[f][u["obase"] + j]) != int(oobj[f][j]):
                        bad.append(f"unit {i} object {j} {f}: gpu {rep.objects[f][u['obase'] + j]} oracle {oobj[f][j]}")
            osh = u["npc"] + len(u["hobjs"])
            for f in shared:
                shared[f] += int(okeys[f][osh])
            for f in glob:
                glob[f] += int(oglob[f])
        gsh = n_pcs + n_obj
        for f in shared:
            if int(rep.keys[f][gsh]) != shared[f]:
                bad.append(f"SHARED {f}: gpu {rep.keys[f][gsh]} sum of units {shared[f]}")
        for f in glob:
            if int(rep.globals[f]) != glob[f]:
                bad.append(f"globals {f}: gpu {rep.globals[f]} sum of units {glob[f]}")
        rep.close()
        assert not bad, f"epoch {rep_i}:\n" + "\n".join(bad[:30])
    ctx.close()
    torch.cuda.synchronize()


def test_units_reject_misaligned(torch_cuda):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    hobjs = W.host_objects(G.FUZZ, 0, 1)
    recs = G.records_host(G.FUZZ, 0, 1, 0, 1001)
    drec = W.device_records(recs)
    ctx = ve.Context(n_pcs=64, max_objects=len(hobjs))
    ctx.set_units([W.device_objects(hobjs)])
    with pytest.raises(ve.VeError):
        ctx.analyze_units([(drec.data_ptr() + 24, 1000, 0, 64)])
    with pytest.raises(ve.VeError):
        ctx.analyze_units([(drec.data_ptr(), 1001, 1, 64)])     # PC range beyond the ctx
    ctx.close()
