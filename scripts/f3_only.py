"""One ve_temporal_loads call on the full cfg2 gemm epoch (for ncu launch lists)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import vegen as G  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

inf = G.info(G.CFG2, 1)
n = inf["n_records"]
recs = torch.empty(n * 24, dtype=torch.uint8, device="cuda")
G.records_device(G.CFG2, 1, G.SEEDS[G.CFG2], 0, n, recs.data_ptr(), torch.cuda.current_stream().cuda_stream)
ctx = ve.Context(n_pcs=inf["n_pcs"], max_objects=8)
ctx.set_objects([dict(o, pre=None, post=None) for o in G.objects(G.CFG2, 1)])
for _ in range(2):
    out = ctx.temporal_loads(recs, n)
print(out[:5].tolist())
