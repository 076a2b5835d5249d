"""Summarise an ncu --csv launch list: one row per launch (name, duration us, metrics), skipping generator kernels."""
import csv
import sys
from collections import OrderedDict

rows = list(csv.reader(open(sys.argv[1])))
skip = sys.argv[2].split(",") if len(sys.argv) > 2 else ["k_snapshot", "k_records", "k_dedup_gen"]
start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
hdr = rows[start]
ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
L = OrderedDict()
for r in rows[start + 1:]:
    if len(r) <= vi:
        continue
    d = L.setdefault(r[0], {"name": r[ki]})
    d[r[mi]] = r[vi].replace(",", "")
for i, d in L.items():
    if any(d["name"].startswith(s) for s in skip):
        continue
    t = float(d.get("gpu__time_duration.sum", 0)) / 1e3
    extra = " ".join(f"{k.split('.')[0].split('__')[-1]}={float(v):.3g}" for k, v in d.items()
                     if k not in ("name", "gpu__time_duration.sum"))
    print(f"{i:>5} {t:10.1f} us  {d['name'][:60]:60s} {extra}")
