"""ncu target: ve_dyadic_fit on the cfg2 gemm epoch records (debug)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import vegen as G  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

cfg, ep, seed = G.CFG2, 1, 2
inf = G.info(cfg, ep)
n = inf["n_records"]
s = torch.cuda.current_stream().cuda_stream
recs = torch.empty(n * 24, dtype=torch.uint8, device="cuda")
G.records_device(cfg, ep, seed, 0, n, recs.data_ptr(), s)
objs = [{k: o[k] for k in ("base", "size", "id", "elem_width")} | {"pre": None, "post": None} for o in G.objects(cfg, ep)]
ctx = ve.Context(n_pcs=inf["n_pcs"], max_objects=len(objs), hist_capacity=1 << 20)
ctx.set_objects(objs)
for _ in range(2):
    out = ctx.dyadic_fit(recs, n, stream=s)
print(out)
