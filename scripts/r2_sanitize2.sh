#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck on cfg1 and a 300 K-record fuzz trace, both K1 kernels
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_sanitizer.log; : > $L
cat > /tmp/san_run.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np
from gen import vegen as G
from oracle import oracle as O
from tests import parity, workloads as W
from paper_conf_asplos_zhouhmm022_b200 import ve
which = sys.argv[1]
if which == "cfg1":
    hobjs = W.host_objects(G.CFG1, 0, 1); recs = G.records_host(G.CFG1, 0, 1, 0, 1 << 20); npcs = 16
else:
    hobjs = W.host_objects(G.FUZZ, 0, 4); recs = G.records_host(G.FUZZ, 0, 4, 0, 300001); npcs = 64
ctx = ve.Context(n_pcs=npcs, max_objects=8, hist_capacity=1 << 20)
ctx.set_objects(W.device_objects(hobjs))
ctx.analyze_records(W.device_records(recs), len(recs))
ctx.snapshot_diff_all()
rep = ctx.report()
okeys, oglob, oobj = O.analyze(O.make_config(npcs), hobjs, recs)
print(which, os.environ.get("VE_K1"), "mismatches", len(parity.compare_with_oracle(rep, okeys, oglob, oobj)))
PY
for k in 1 2; do for w in cfg1 fuzz; do for tool in memcheck racecheck synccheck; do
  echo "== VE_K1=$k $w $tool" >> $L
  VE_K1=$k timeout 900 compute-sanitizer --tool $tool --print-limit 10 python /tmp/san_run.py $w 2>&1 | grep -v "^\s*$" | tail -6 >> $L
done; done; done
