"""Per-kernel time shares of an ncu launch list (--metrics gpu__time_duration.sum --csv)."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h = [r for r in rows if r and "Kernel Name" in r][0]
hi = rows.index(h)
ki, vi = h.index("Kernel Name"), h.index("Metric Value")
mi = h.index("Metric Name") if "Metric Name" in h else None
hdr = sys.argv[2] if len(sys.argv) > 2 else "bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-f1 --no-cfg5 (2 steps: warm-up + timed)"
d, n = collections.Counter(), collections.Counter()
for r in rows[hi + 1:]:
    if len(r) < len(h):
        continue
    if mi is not None and r[mi] != "gpu__time_duration.sum":
        continue
    k = r[ki].split("(")[0]
    d[k] += float(r[vi].replace(",", ""))
    n[k] += 1
gen = {k for k in d if not k.startswith("ve::") and not k.startswith("void ve::")}   # input generator (untimed)
tot = sum(v for k, v in d.items() if k not in gen)
print("# ncu launch list (gpu__time_duration.sum, --clock-control none), " + hdr + "\n# cold-cache serialised per-launch"
      " times: compare SHARES, not absolutes; shares are of the libve kernels (the step)")
print(f"{'ms':>10} launches  share  kernel")
for k, v in d.most_common():
    if k not in gen:
        print(f"{v / 1e6:10.3f} {n[k]:8d} {100 * v / tot:5.1f}%  {k}")
print(f"total {tot / 1e6:.3f} ms (libve)")
for k in sorted(gen):
    print(f"# input generator, outside the timed region: {k} {d[k] / 1e6:.3f} ms x {n[k]}")
