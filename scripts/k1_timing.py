"""A/B timing of K1 on full-size epochs: analyze (CUDA events) and report (wall, synchronised).
usage: python scripts/k1_timing.py [cfg2,cfg3,cfg4e0,cfg4e1 ...]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import vegen as G  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

PLANS = {"cfg2": (G.CFG2, 1, 2, 1 << 22), "cfg2e0": (G.CFG2, 0, 2, 1 << 22),
         "cfg3": (G.scaled(G.CFG3, 0), 0, 3, 1 << 25),
         "cfg4e0": (G.scaled(G.CFG4, 0), 0, 4, 1 << 22), "cfg4e1": (G.scaled(G.CFG4, 0), 1, 4, 1 << 22)}
which = sys.argv[1].split(",") if len(sys.argv) > 1 else ["cfg2", "cfg4e0", "cfg4e1"]
reps = int(os.environ.get("REPS", "3"))
st = torch.cuda.current_stream()
sp = st.cuda_stream
for name in which:
    cfg, epoch, seed, hcap = PLANS[name]
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
    an, rp = [], []
    for it in range(reps):
        ctx.set_objects(dobjs)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        ctx.analyze_records(recs, n, stream=sp)
        b.record(st)
        torch.cuda.synchronize()
        an.append(a.elapsed_time(b))
        t0 = time.perf_counter()
        rep = ctx.report()
        torch.cuda.synchronize()
        rp.append(1e3 * (time.perf_counter() - t0))
    k = rep.keys
    sig = (int(k["n_ld"].sum()), int(k["n_st_eq_pre"].sum()), int(k["n_distinct"].sum()), int(k["line_state"].sum()))
    print(f"{name:7s} n={n} analyze_ms={min(an):8.3f} report_ms={min(rp):8.3f} rec/s={n / min(an) * 1e3:.3e} sig={sig}",
          flush=True)
    ctx.close()
    del dobjs, recs
    torch.cuda.empty_cache()
