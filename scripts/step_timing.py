"""Per-call wall timing of one bench step (debug; each call bracketed by a device sync)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

torch.cuda.set_device(0)
wl = bench.Workload(0, 1, torch.device("cuda", 0))
ctx = ve.Context(n_pcs=5, max_objects=8, hist_capacity=1 << 22, device=0)
s = torch.cuda.current_stream()


def t(name, fn):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    r = fn()
    torch.cuda.synchronize()
    print(f"{name:28s} {1e3 * (time.perf_counter() - t0):9.3f} ms", flush=True)
    return r


for it in range(3):
    print("-- step", it)
    for ep, e in enumerate(wl.epochs):
        t(f"set_objects[{ep}]", lambda: ctx.set_objects(e["objs"]))
        t(f"analyze[{ep}]", lambda: ctx.analyze_records(e["recs"], e["n"], stream=s.cuda_stream))
        t(f"diff[{ep}]", lambda: ctx.snapshot_diff(2, stream=s.cuda_stream))
        t(f"report[{ep}]", lambda: ctx.report())
    t("dedup", lambda: ctx.object_dedup(wl.dedup_objs(), stream=s.cuda_stream))
