#!/bin/bash
# MOMENT_SCAN_PREFETCH 0 / 1 on C2 (C1 beside it), interleaved; parity with it on.
mkdir -p gpurun_out/exp4
for r in 1 2 3; do for p in 0 1; do
  MOMENT_SCAN_PREFETCH=$p timeout 300 python bench.py --no-cpu-baseline > gpurun_out/exp4/b.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/exp4/b.json'));print('C2 scan_prefetch=$p r=$r',round(d['value']/1e6,3),round(d['ms_per_step']*1e3,2),round(d['roofline']['frac'],3))" >> gpurun_out/exp4/summary.txt 2>&1
done; done
for p in 0 1; do
  MOMENT_SCAN_PREFETCH=$p timeout 300 python bench.py --config C1 --no-cpu-baseline > gpurun_out/exp4/b.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/exp4/b.json'));print('C1 scan_prefetch=$p',round(d['value']/1e6,3),round(d['ms_per_step']*1e3,2))" >> gpurun_out/exp4/summary.txt 2>&1
done
MOMENT_SCAN_PREFETCH=1 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -1 >> gpurun_out/exp4/summary.txt
