"""Per-source-line STL/LDL counts of one kernel in a cubin (nvdisasm -g)."""
import collections
import re
import subprocess
import sys

cubin, kern = sys.argv[1], sys.argv[2]
out = subprocess.run(["nvdisasm", "-g", cubin], capture_output=True, text=True).stdout.splitlines()
sec = None
cur = None
cnt = collections.Counter()
tot = 0
for l in out:
    if l.startswith(".text."):
        sec = l
        continue
    m = re.search(r'//## File "(.*?)", line (\d+)', l)
    if m:
        cur = (m.group(1).split("/")[-1], int(m.group(2)))
        continue
    if sec and kern in sec and re.search(r"\b(STL|LDL)", l):
        cnt[cur] += 1
        tot += 1
print("total", tot)
for k, v in cnt.most_common(int(sys.argv[3]) if len(sys.argv) > 3 else 25):
    print(k, v)
