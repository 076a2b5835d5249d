import sys, os
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "."))
import torch, bench
from paper_conf_asplos_zhouhmm022_b200 import ve
torch.cuda.set_device(0)
wl = bench.Workload(0, 1, torch.device("cuda", 0))
ctx = ve.Context(n_pcs=5, max_objects=8, hist_capacity=1 << 23)
for e in wl.epochs:
    ctx.set_objects(e["objs"]); ctx.analyze_records(e["recs"], e["n"]); r = ctx.report()
    print("n_distinct per key:", [int(x) for x in r.keys["n_distinct"]], "PC sum", int(r.keys["n_distinct"][:5].sum()))
