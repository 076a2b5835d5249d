"""Per-source-line instruction and stall shares of one kernel in an ncu report
(usage: ncu_lines.py report.ncu-rep [n_units] [top])."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
units = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr = next(r for r in rows if r and r[0] == "Line No")
iS = hdr.index("Warp Stall Sampling (All Samples)")
iI = hdr.index("Instructions Executed")
fname = None
res = []
for r in rows:
    if len(r) >= 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if len(r) < len(hdr) or r[0] in ("Line No", ""):
        continue
    try:
        res.append((int(r[iI]) if r[iI] != "-" else 0, int(r[iS]) if r[iS] != "-" else 0, fname, r[0], r[1][:100]))
    except ValueError:
        pass
ti = sum(x[0] for x in res) or 1
ts = sum(x[1] for x in res) or 1
print(f"total warp instructions {ti}  ({ti / units:.1f} per unit)  stall samples {ts}")
for i, s, f, l, src in sorted(res, reverse=True)[:top]:
    print(f"{i / units:7.1f}/u {100 * i / ti:5.1f}% inst {100 * s / ts:5.1f}% stall {f[:16]}:{l} {src}")
