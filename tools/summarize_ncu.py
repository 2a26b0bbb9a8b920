"""Summarise an `ncu --page raw --csv` export: one line per kernel launch with the key metrics."""
import csv
import sys


def main(path):
    lines = [l for l in open(path) if l.startswith('"')]
    rows = list(csv.reader(lines))
    head, units, data = rows[0], rows[1], rows[2:]
    want = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "lts__t_bytes.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
            "launch__grid_size", "launch__registers_per_thread"]
    idx = [head.index(w) if w in head else None for w in want]
    short = ["kernel", "time", "dram_rd", "dram_wr", "l2_bytes", "dram%", "occ%", "sm%", "grid", "regs"]
    print(" | ".join(short))
    for r in data:
        vals = []
        for w, i in zip(want, idx):
            if i is None:
                vals.append("-")
                continue
            v = r[i]
            if w == "Kernel Name":
                v = v.replace("(anonymous namespace)::", "").replace("moment::", "").replace("void ", "").split("(")[0][:28]
            else:
                u = units[i]
                vals_u = f"{v} {u}".strip()
                v = vals_u
            vals.append(v)
        print(" | ".join(vals))


if __name__ == "__main__":
    main(sys.argv[1])
