#!/bin/bash
# ncu full capture of k_analyze on cfg4 epoch 0 and epoch 1 (full size), source-level
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
cat > /tmp/c4one.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import torch
from gen import vegen as G
from paper_conf_asplos_zhouhmm022_b200 import ve
ep = int(sys.argv[1]); cfg = G.scaled(G.CFG4, 0); sp = torch.cuda.current_stream().cuda_stream
inf = G.info(cfg, ep); n = inf["n_records"]; dobjs = []
for i, o in enumerate(G.objects(cfg, ep)):
    d = {k: o[k] for k in ("base", "size", "id", "elem_width")}
    for side in ("pre", "post"):
        t = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
        G.snapshot_device(cfg, ep, 4, i, side == "post", t.data_ptr(), sp); d[side] = t
    dobjs.append(d)
recs = torch.empty(n * 24, dtype=torch.uint8, device="cuda"); G.records_device(cfg, ep, 4, 0, n, recs.data_ptr(), sp)
ctx = ve.Context(n_pcs=inf["n_pcs"], max_objects=len(dobjs), hist_capacity=1 << 22)
ctx.set_objects(dobjs); ctx.analyze_records(recs, n, stream=sp); ctx.report()
PY
for ep in 0 1; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_analyze -c 1 -f \
   -o gpurun_out/r2_prof_c4e$ep python /tmp/c4one.py $ep > gpurun_out/r2_prof_c4e$ep.log 2>&1
echo "ep $ep exit $?" >> gpurun_out/r2_prof_c4e$ep.log
done
