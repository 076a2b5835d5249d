"""Time one cfg5 units batch: set_units / analyze_units / report (usage: units_probe.py [n_kernels] [first])."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import vegen as G  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

K = int(sys.argv[1]) if len(sys.argv) > 1 else 250
k0 = int(sys.argv[2]) if len(sys.argv) > 2 else 0
cfg, seed = G.scaled(G.CFG5, 0), 5
sp = torch.cuda.current_stream().cuda_stream
ks = list(range(k0, k0 + K))
infos = {k: G.info(cfg, k) for k in ks}
tot = sum(infos[k]["n_records"] + (infos[k]["n_records"] & 1) for k in ks)
recs = torch.empty(tot * 24, dtype=torch.uint8, device="cuda")
uobjs, units, pcb, ob, r0 = [], [], 0, 0, 0
keep = []
for k in ks:
    n = infos[k]["n_records"]
    G.records_device(cfg, k, seed, 0, n, recs.data_ptr() + r0 * 24, sp)
    objs = []
    for i, o in enumerate(G.objects(cfg, k)):
        d = {f: o[f] for f in ("base", "size", "elem_width")}
        d["id"] = o["id"] + ob
        for side in ("pre", "post"):
            t = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
            G.snapshot_device(cfg, k, seed, i, side == "post", t.data_ptr(), sp)
            d[side] = t
        objs.append(d)
    uobjs.append(objs)
    units.append((recs.data_ptr() + r0 * 24, n, pcb, infos[k]["n_pcs"]))
    pcb += infos[k]["n_pcs"]
    ob += len(objs)
    r0 += n + (n & 1)
print(f"{K} kernels, {sum(u[1] for u in units)} records, {pcb} PCs, {ob} objects", flush=True)
ctx = ve.Context(n_pcs=pcb, max_objects=ob, hist_capacity=1 << 25)
for it in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    ctx.set_units(uobjs)
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    ctx.analyze_units(units)
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    rep = ctx.report()
    t3 = time.perf_counter()
    print(f"it {it}: set {1e3*(t1-t0):.2f} ms analyze {1e3*(t2-t1):.2f} ms report {1e3*(t3-t2):.2f} ms "
          f"n_records {int(rep.globals['n_records'])} hist_entries {int(rep.globals['hist_entries'])}", flush=True)
    rep.close()
ctx.close()
