"""k_analyze time vs record count (gemm-epoch prefixes): fixed cost vs per-record cost."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

torch.cuda.set_device(0)
wl = bench.Workload(0, 1, torch.device("cuda", 0))
ctx = ve.Context(n_pcs=5, max_objects=8, hist_capacity=1 << 23, device=0)
s = torch.cuda.current_stream()
e = wl.epochs[1]
ctx.set_objects(e["objs"])
N = e["n"]
for n in [0, 1 << 16, 1 << 20, 1 << 22, 1 << 24, 1 << 26, N // 2, N]:
    ts = []
    for it in range(4):
        ctx.reset()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record(s)
        ctx.analyze_records(e["recs"], n, stream=s.cuda_stream)
        b.record(s)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    t = min(ts[1:])
    print(f"n={n:>11d}  {t:8.3f} ms  {n / max(t, 1e-9) / 1e6:8.2f} G rec/s", flush=True)
