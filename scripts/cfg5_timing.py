"""Per-call wall timing of cfg5 kernels (debug; each call bracketed by a device sync)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import vegen as G  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

cfg, seed = G.scaled(G.CFG5, 0), 5
s = torch.cuda.current_stream()
sp = s.cuda_stream
ctx = ve.Context(n_pcs=64, max_objects=4, hist_capacity=1 << 23)
kernels = [int(x) for x in sys.argv[1:]] or list(range(0, 4000, 200))


def t(fn):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    r = fn()
    torch.cuda.synchronize()
    return r, 1e3 * (time.perf_counter() - t0)


for rep in range(2):
    for k in kernels:
        inf = G.info(cfg, k)
        n = inf["n_records"]
        dobjs = []
        for i, o in enumerate(G.objects(cfg, k)):
            d = {f: o[f] for f in ("base", "size", "id", "elem_width")}
            for side in ("pre", "post"):
                tt = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
                G.snapshot_device(cfg, k, seed, i, side == "post", tt.data_ptr(), sp)
                d[side] = tt
            dobjs.append(d)
        recs = torch.empty(n * 24, dtype=torch.uint8, device="cuda")
        G.records_device(cfg, k, seed, 0, n, recs.data_ptr(), sp)
        _, a = t(lambda: ctx.set_objects(dobjs))
        _, b = t(lambda: ctx.analyze_records(recs, n, stream=sp))
        r, c = t(lambda: ctx.report())
        r.close()
        if rep == 1:
            print(f"k {k:4d} n {n:8d} pcs {inf['n_pcs']:2d} obj {inf['n_obj']} set {a:7.3f} analyze {b:7.3f} "
                  f"report {c:7.3f} ms", flush=True)
