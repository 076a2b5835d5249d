"""Summarise an ncu report: key metrics + top source lines by stall samples / executed instructions."""
import csv
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(raw.splitlines()))
h, u, v = rows[0], rows[1], rows[2]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__inst_executed.sum", "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "l1tex__throughput.avg.pct_of_peak_sustained_active"]
for i, n in enumerate(h):
    if n in want:
        print(f"{n:60s} {v[i]:>20s} {u[i]}")
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
        res.append((int(r[iex] or 0), int(r[iss] or 0), r[0], r[1][:100]))
    except ValueError:
        pass
tot = sum(o[0] for o in res) or 1
ts = sum(o[1] for o in res) or 1
print(f"source-attributed instructions {tot}  stall samples {ts}")
print("-- top lines by stall samples")
for o in sorted(res, key=lambda x: -x[1])[:top]:
    print(f"{o[0]:>11} {100*o[0]/tot:5.1f}%i s={o[1]:>7} {100*o[1]/ts:5.1f}%s L{o[2]:>4} {o[3]}")
