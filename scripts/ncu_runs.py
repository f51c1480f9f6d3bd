"""Group the SASS of one ncu capture into runs of equal execution count (basic blocks) and
print the heaviest: python scripts/ncu_runs.py rep.ncu-rep [n]"""
import csv
import subprocess
import sys

f = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(['ncu', '-i', f, '--page', 'source', '--csv', '--print-source', 'sass'],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = rows[1]
data = rows[2:]
iS = hdr.index('Warp Stall Sampling (All Samples)')
iI = hdr.index('Instructions Executed')
iSrc = hdr.index('Source')
runs, cur = [], None
for i, r in enumerate(data):
    c = int(r[iI]) if r[iI].isdigit() else 0
    s = int(r[iS]) if r[iS].isdigit() else 0
    if cur and cur[2] == c:
        cur[1] = i
        cur[3] += c
        cur[4] += s
    else:
        cur = [i, i, c, c, s]
        runs.append(cur)
tot = sum(r[3] for r in runs)
tots = sum(r[4] for r in runs)
print(f"instructions {tot}  samples {tots}")
for r in sorted(runs, key=lambda r: -r[3])[:n]:
    print(f"{r[0]:5d}-{r[1]:5d} exec={r[2]:10d} inst%={r[3] / tot * 100:5.1f} stall%={r[4] / tots * 100:5.1f}  "
          f"{data[r[0]][iSrc][:60]}")
