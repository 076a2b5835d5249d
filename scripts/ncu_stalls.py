"""Top SASS instructions of an ncu report per stall reason
(usage: ncu_stalls.py report.ncu-rep [reason ...])."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
reasons = sys.argv[2:] or ["stall_long_sb", "stall_wait", "stall_barrier", "stall_branch_resolving", "stall_short_sb"]
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr = next(r for r in rows if r and "Address" in r)
body = [r for r in rows if len(r) == len(hdr) and r[0] not in ("Address", "")]
for reason in reasons:
    i = hdr.index(reason)
    vals = []
    for r in body:
        try:
            vals.append((int(r[i]), r[0][-5:], r[1][:70]))
        except ValueError:
            pass
    tot = sum(v[0] for v in vals) or 1
    print(f"== {reason}: {tot} samples")
    for v, a, src in sorted(vals, reverse=True)[:8]:
        print(f"  {100 * v / tot:5.1f}% {a} {src}")
