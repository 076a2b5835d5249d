"""Top source lines of an ncu report by executed instructions (per window if a window count is given)."""
import csv
import subprocess
import sys

rep = sys.argv[1]
nwin = float(sys.argv[2]) if len(sys.argv) > 2 else 0
top = int(sys.argv[3]) if len(sys.argv) > 3 else 60
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(src.splitlines()))
hi = [i for i, r in enumerate(rows[:10]) if "Instructions Executed" in r][0]
h = rows[hi]
iex, iss = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
res = []
for r in rows[hi + 1:]:
    if len(r) < len(h) or not r[0]:
        continue
    try:
        res.append((int(r[iex] or 0), int(r[iss] or 0), r[0], r[1][:110]))
    except ValueError:
        pass
tot = sum(o[0] for o in res) or 1
print(f"total {tot}" + (f"  per window {tot / nwin:.1f}" if nwin else ""))
for o in sorted(res, key=lambda x: -x[0])[:top]:
    pw = f"{o[0] / nwin:6.2f}/w" if nwin else ""
    print(f"{o[0]:>11} {pw} {100*o[0]/tot:5.1f}% L{o[2]:>4} {o[3]}")
