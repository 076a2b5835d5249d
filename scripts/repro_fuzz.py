"""Repro: one FUZZ trace through libve vs the oracle (debug / sanitizer runs)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from gen import vegen as G  # noqa: E402
from oracle import oracle as O  # noqa: E402
from tests import parity, workloads as W  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

seed = int(sys.argv[1]) if len(sys.argv) > 1 else 4
n = int(sys.argv[2]) if len(sys.argv) > 2 else 300001
npcs = int(sys.argv[3]) if len(sys.argv) > 3 else 64
hobjs = W.host_objects(G.FUZZ, 0, seed)
recs = G.records_host(G.FUZZ, 0, seed, 0, n)
if npcs == 5:
    pc = recs["pc"].astype(np.int64)
    recs["pc"] = np.where(pc < 64, pc % 5, 5 + (pc - 64)).astype(np.uint32)
ctx = ve.Context(n_pcs=npcs, max_objects=8, hist_capacity=1 << 20)
ctx.set_objects(W.device_objects(hobjs))
ctx.analyze_records(W.device_records(recs), n)
rep = ctx.report()
okeys, oglob, oobj = O.analyze(O.make_config(npcs), hobjs, recs)
bad = parity.compare_with_oracle(rep, okeys, oglob, oobj)
print("mismatches", len(bad))
for b in bad[:20]:
    print(b)
