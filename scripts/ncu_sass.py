"""SASS of one kernel in an ncu report with per-instruction execution counts per unit,
in address order (usage: ncu_sass.py report.ncu-rep n_units [min_per_unit])."""
import csv
import io
import subprocess
import sys

rep, units = sys.argv[1], float(sys.argv[2])
thr = float(sys.argv[3]) if len(sys.argv) > 3 else 0.5
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr = next(r for r in rows if r and "Address" in r)
iA, iS = hdr.index("Address"), hdr.index("Source")
iI = hdr.index("Instructions Executed")
iW = hdr.index("Warp Stall Sampling (All Samples)")
tot = 0
for r in rows:
    if len(r) < len(hdr) or r[iA] in ("Address", ""):
        continue
    try:
        n = int(r[iI])
    except ValueError:
        continue
    tot += n
    if n / units >= thr:
        print(f"{r[iA][-5:]} {n / units:6.2f} {r[iW]:>6s}  {r[iS][:90]}")
print("total per unit", tot / units)
