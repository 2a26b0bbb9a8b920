"""Print the key rows of `ncu --page details --csv` (stdin): duration, throughput, occupancy, stalls."""
import csv
import sys

KEEP = ("Duration", "Memory Throughput", "DRAM Throughput", "L2 Hit Rate", "Achieved Occupancy",
        "Theoretical Occupancy", "Registers Per Thread", "Issued Warp Per Scheduler", "No Eligible",
        "Eligible Warps Per Scheduler", "Warp Cycles Per Issued Instruction", "Grid Size", "Block Size",
        "L1/TEX Hit Rate", "Mem Busy", "Max Bandwidth", "Compute (SM) Throughput")
rows = list(csv.reader(l for l in sys.stdin if l.startswith('"')))
head = rows[0]
ni, si, mi, ui, vi = (head.index(x) for x in ("Kernel Name", "Section Name", "Metric Name", "Metric Unit", "Metric Value"))
for r in rows[1:]:
    if r[mi] in KEEP:
        print(f"{r[si][:28]:28s} {r[mi]:40s} {r[vi]:>14s} {r[ui]}")
    if r[mi] == "" and len(r) > vi + 2 and "stall" in r[vi + 1].lower():
        print("  >>", r[vi + 2][:300])
