"""Summarise an ncu --csv launch list: per-kernel count, total and mean device time."""
import csv
import sys
from collections import defaultdict


def main(path):
    rows = []
    with open(path) as f:
        lines = [l for l in f if l.startswith('"')]
    rd = csv.DictReader(lines)
    tot = defaultdict(float)
    cnt = defaultdict(int)
    for r in rd:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = r["Kernel Name"].split("(")[0].split("<")[0]
        name = name.replace("moment::", "").replace("(anonymous namespace)::", "")
        v = float(r["Metric Value"].replace(",", ""))
        unit = r.get("Metric Unit", "nsecond")
        if unit in ("usecond", "us"):
            v *= 1e3
        elif unit in ("msecond", "ms"):
            v *= 1e6
        tot[name] += v
        cnt[name] += 1
    allt = sum(tot.values())
    print(f"{'kernel':40s} {'launches':>8s} {'total_us':>10s} {'mean_us':>9s} {'share':>6s}")
    for k in sorted(tot, key=lambda k: -tot[k]):
        print(f"{k[:40]:40s} {cnt[k]:8d} {tot[k] / 1e3:10.1f} {tot[k] / cnt[k] / 1e3:9.2f} {tot[k] / allt:6.1%}")


if __name__ == "__main__":
    main(sys.argv[1])
