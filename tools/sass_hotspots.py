"""Top SASS instructions by warp-stall samples, per kernel, from
`ncu -i X --page source --csv --print-source sass` (all kernels of the report, one block each).

    python tools/sass_hotspots.py report.csv [top_n] [kernel_substring] [which_match]
"""
import csv
import sys


def blocks(path):
    cur, name = None, None
    for r in csv.reader(open(path)):
        if r and r[0] == "Kernel Name":
            if cur:
                yield name, cur
            name, cur = r[1], []
        elif cur is not None:
            cur.append(r)
    if cur:
        yield name, cur


def main():
    path = sys.argv[1]
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
    sub = sys.argv[3] if len(sys.argv) > 3 else ""
    which = int(sys.argv[4]) if len(sys.argv) > 4 else -1
    matches = [(k, b) for k, b in blocks(path) if sub in k]
    for j, (name, rows) in enumerate(matches):
        if which >= 0 and j != which:
            continue
        h = rows[0]
        si = h.index("Warp Stall Sampling (All Samples)")
        data = [r for r in rows[1:] if len(r) > si and r[si].strip().isdigit()]
        tot = sum(int(r[si]) for r in data) or 1
        print(f"== {name[:100]}  ({tot} samples, {len(data)} instructions)")
        for i, r in sorted(enumerate(data), key=lambda x: -int(x[1][si]))[:n]:
            print(f"{int(r[si]) / tot * 100:5.1f}%  [{i:4d}] {r[1].strip()[:90]}")


if __name__ == "__main__":
    main()
