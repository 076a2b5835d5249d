"""Per-phase wall timing (device-synchronised) of full-size cfg3 / cfg4 epochs (debug)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import vegen as G  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

which = sys.argv[1] if len(sys.argv) > 1 else "both"
plans = [("cfg3", G.scaled(G.CFG3, 0), 0, 3, 1 << 25), ("cfg4", G.scaled(G.CFG4, 0), 0, 4, 1 << 22),
         ("cfg4", G.scaled(G.CFG4, 0), 1, 4, 1 << 22)]
sp = torch.cuda.current_stream().cuda_stream


def t(name, fn):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    r = fn()
    torch.cuda.synchronize()
    print(f"{name:34s} {1e3 * (time.perf_counter() - t0):9.3f} ms", flush=True)
    return r


for name, cfg, epoch, seed, hcap in plans:
    if which != "both" and which != name:
        continue
    inf = G.info(cfg, epoch)
    n = inf["n_records"]
    dobjs = []
    for i, o in enumerate(G.objects(cfg, epoch)):
        d = {k: o[k] for k in ("base", "size", "id", "elem_width")}
        for side in ("pre", "post"):
            tt = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
            G.snapshot_device(cfg, epoch, seed, i, side == "post", tt.data_ptr(), sp)
            d[side] = tt
        dobjs.append(d)
    recs = torch.empty(n * 24, dtype=torch.uint8, device="cuda")
    G.records_device(cfg, epoch, seed, 0, n, recs.data_ptr(), sp)
    ctx = ve.Context(n_pcs=inf["n_pcs"], max_objects=len(dobjs), hist_capacity=hcap)
    print(f"== {name} epoch {epoch}: {n} records, {len(dobjs)} objects, {inf['n_pcs']} pcs")
    for it in range(2):
        t(f"set_objects", lambda: ctx.set_objects(dobjs))
        t(f"analyze", lambda: ctx.analyze_records(recs, n, stream=sp))
        t(f"report", lambda: ctx.report())
    ctx.close()
    del dobjs, recs
    torch.cuda.empty_cache()
