"""GPU-side test helpers: run libve.so on seeded inputs and compare with the CPU
oracle (test infrastructure; the product is reached only through its binding)."""
import numpy as np

from oracle import oracle as O
from tests import parity, workloads as W


def _ve():
    from paper_conf_asplos_zhouhmm022_b200 import ve
    return ve


def _run_gpu(torch_cuda, n_pcs, hobjs, recs, chunks=None, topk=8, hist_capacity=1 << 20, diff_modes=()):
    ve = _ve()
    dobjs = W.device_objects(hobjs)
    ctx = ve.Context(n_pcs=n_pcs, max_objects=max(len(hobjs), 1), topk=topk, hist_capacity=hist_capacity)
    ctx.set_objects(dobjs)
    drec = W.device_records(recs)
    n = len(recs)
    if chunks is None:
        ctx.analyze_records(drec, n)
    else:
        bounds = [0] + list(chunks) + [n]
        for a, b in zip(bounds[:-1], bounds[1:]):
            if b > a:
                ctx.analyze_records(drec[a * 24:b * 24], b - a)
    rep = ctx.report()
    diffs = {}
    for oid, mode, mask in diff_modes:
        dm = torch_cuda.from_numpy(mask).cuda() if mask is not None else None
        diffs[(oid, mode)] = ctx.snapshot_diff(oid, mode, dm)
    ctx.close()
    return rep, diffs


def _check(torch_cuda, n_pcs, hobjs, recs, **kw):
    cfg = O.make_config(n_pcs, topk=kw.get("topk", 8))
    okeys, oglob, oobj = O.analyze(cfg, hobjs, recs)
    modes = []
    for o in hobjs:
        if o.get("pre") is not None and o.get("post") is not None:
            ne = (o["size"] + o["elem_width"] - 1) // o["elem_width"]
            mask = np.random.default_rng(o["id"]).integers(0, 1 << 32, (ne + 31) // 32, dtype=np.uint64).astype(np.uint32)
            modes += [(o["id"], O.DIFF_WRITTEN, None), (o["id"], O.DIFF_ALL, None), (o["id"], O.DIFF_MASK, mask)]
    rep, diffs = _run_gpu(torch_cuda, n_pcs, hobjs, recs, diff_modes=modes, **kw)
    bad = parity.compare_with_oracle(rep, okeys, oglob, oobj)
    for (oid, mode), gd in diffs.items():
        mask = [m for (i, md, m) in modes if i == oid and md == mode][0]
        od = O.snapshot_diff(cfg, hobjs, recs, oid, mode, mask)
        bad += [f"obj {oid} mode {mode} " + s for s in parity.compare_diff(gd, od)]
    assert not bad, "\n".join(bad[:40])
    return rep, okeys
