#!/bin/bash
# ncu of the tiered gather (C4 shape: HBM cache + pinned-host rows read zero-copy over PCIe): DRAM and PCIe
# bytes, duration and occupancy of a few gather launches of tools/results_matrix.py.
OUT=${1:-gpurun_out/ncu_tiered_C4}
ncu --clock-control none -k "regex:gather_kernel" -s 2 -c 3 \
    --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,pcie__read_bytes.sum,pcie__write_bytes.sum,sm__warps_active.avg.pct_of_peak_sustained_active,launch__grid_size \
    --csv --log-file "$OUT.csv" \
    python tools/results_matrix.py --configs C4 --batches 24 --lanes 1 --oracle-s 0.1 --presample 64 > /dev/null 2>&1
cat "$OUT.csv" | grep -v "^==" | python -c "
import csv, sys
rows = list(csv.DictReader(sys.stdin))
for r in rows:
    print(r['Kernel Name'][:40], '|', r['Metric Name'], '|', r['Metric Value'], r['Metric Unit'])
"
