#!/bin/bash
# Gather L2 hints (MOMENT_GATHER_L2 "<load><store>": 0 normal, 1 evict_first, 2 evict_last) with the indptr prefetch on, C2.
mkdir -p gpurun_out/exp3
for r in 1 2; do for p in 01 11 00 10; do
  MOMENT_GATHER_L2=$p timeout 300 python bench.py --no-cpu-baseline > gpurun_out/exp3/b.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/exp3/b.json'));print('L2=$p r=$r',round(d['value']/1e6,3),round(d['ms_per_step']*1e3,2),round(d['roofline']['frac'],3))" >> gpurun_out/exp3/summary.txt 2>&1
done; done
