"""f1 record intervals on the cfg2 gemm epoch (225.6 M records): CUDA-event time of ve_record_intervals."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from gen import vegen as G  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

cfg, epoch, seed = G.CFG2, 1, 2
inf = G.info(cfg, epoch)
n = inf["n_records"]
sp = torch.cuda.current_stream().cuda_stream
recs = torch.empty(n * 24, dtype=torch.uint8, device="cuda")
G.records_device(cfg, epoch, seed, 0, n, recs.data_ptr(), sp)
ctx = ve.Context(n_pcs=inf["n_pcs"], max_objects=8)
ctx.set_objects([{k: o[k] for k in ("base", "size", "id", "elem_width")} for o in G.objects(cfg, epoch)])
out = torch.empty(n * 16, dtype=torch.uint8, device="cuda")
ts = []
for it in range(4):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    a.record()
    k = ctx.record_intervals(recs, n, out)
    b.record()
    torch.cuda.synchronize()
    ts.append(a.elapsed_time(b))
print(f"f1 n={n} merged={k} ms={min(ts):.3f} frac={n * 24 / (min(ts) / 1e3) / 1e9 / 6524.6:.3f}", flush=True)
