"""Top SASS instructions by warp-stall samples from `ncu -i X --page source --csv --print-source sass`."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
si = h.index("Warp Stall Sampling (All Samples)")
data = [r for r in rows[2:] if len(r) > si and r[si].strip().isdigit()]
tot = sum(int(r[si]) for r in data) or 1
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
for i, r in sorted(enumerate(data), key=lambda x: -int(x[1][si]))[:n]:
    # show the instruction with its two predecessors for context
    print(f"{int(r[si]) / tot * 100:5.1f}%  [{i:4d}] {r[1].strip()[:90]}")
