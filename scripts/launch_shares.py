"""Per-kernel time shares of an ncu launch list (--metrics gpu__time_duration.sum --csv)."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h = [r for r in rows if r and "Kernel Name" in r][0]
hi = rows.index(h)
ki, vi = h.index("Kernel Name"), h.index("Metric Value")
d, n = collections.Counter(), collections.Counter()
for r in rows[hi + 1:]:
    if len(r) < len(h):
        continue
    k = r[ki].split("(")[0]
    d[k] += float(r[vi].replace(",", ""))
    n[k] += 1
tot = sum(d.values())
print("# ncu launch list (gpu__time_duration.sum, --clock-control none), bench.py --steps 1 --warmup 1"
      " (2 steps: warm-up + timed)\n# cold-cache serialised per-launch times: compare SHARES, not absolutes")
print(f"{'ms':>10} launches  share  kernel")
for k, v in d.most_common():
    print(f"{v / 1e6:10.3f} {n[k]:8d} {100 * v / tot:5.1f}%  {k}")
print(f"total {tot / 1e6:.3f} ms")
