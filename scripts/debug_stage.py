"""Debug helper: run one fuzz case stage by stage with syncs and timings.
usage: python scripts/debug_stage.py SEED N [stage...]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import vegen as G  # noqa: E402
from tests import workloads as W  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

seed, n = int(sys.argv[1]), int(sys.argv[2])
cfgid = int(os.environ.get("CFG", G.FUZZ))
npcs = G.info(cfgid)["n_pcs"]
hobjs = W.host_objects(cfgid, 0, seed)
recs = G.records_host(cfgid, 0, seed, 0, n)
dobjs = W.device_objects(hobjs)
drec = W.device_records(recs)
torch.cuda.synchronize()
ctx = ve.Context(n_pcs=npcs, max_objects=8, hist_capacity=1 << 20)
ctx.set_objects(dobjs)
t = time.time()
ctx.analyze_records(drec, n)
torch.cuda.synchronize()
print(f"analyze ok {time.time() - t:.3f}s", flush=True)
t = time.time()
rep = ctx.report()
print(f"report ok {time.time() - t:.3f}s", flush=True)
for o in hobjs:
    if o["pre"] is not None and o["post"] is not None:
        d = ctx.snapshot_diff(o["id"], ve.DIFF_ALL)
        print("diff", o["id"], d, flush=True)
