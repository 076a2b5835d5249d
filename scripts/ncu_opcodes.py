"""SASS opcode histogram (executed warp instructions) of an ncu report, per unit of work."""
import collections
import csv
import io
import subprocess
import sys

rep, units = sys.argv[1], float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr = next(r for r in rows if r and "Address" in r)
body = [r for r in rows if len(r) == len(hdr) and r[0] not in ("Address", "")]
ie = hdr.index("Instructions Executed")
c = collections.Counter()
for r in body:
    try:
        n = int(r[ie] or 0)
    except ValueError:
        continue
    t = r[1].split()
    if not t:
        continue
    op = t[1] if t[0].startswith("@") and len(t) > 1 else t[0]
    c[op.split(".")[0]] += n
tot = sum(c.values())
print(f"total {tot / units:.1f} per unit")
for k, v in c.most_common(int(sys.argv[3]) if len(sys.argv) > 3 else 30):
    print(f"{k:10s} {v / units:8.2f} {100 * v / tot:5.1f}%")
