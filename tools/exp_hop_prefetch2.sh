#!/bin/bash
# MOMENT_HOP_PREFETCH 0 / 1 (evict_last) / 2 (no hint) on C2 and C3, interleaved.
mkdir -p gpurun_out/exp2
for cfg in C2 C3; do for r in 1 2; do for p in 0 1 2; do
  MOMENT_HOP_PREFETCH=$p timeout 300 python bench.py --config $cfg --no-cpu-baseline > gpurun_out/exp2/b.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/exp2/b.json'));print('$cfg p=$p r=$r',round(d['value']/1e6,3),round(d['ms_per_step']*1e3,2))" >> gpurun_out/exp2/summary.txt 2>&1
done; done; done
MOMENT_HOP_PREFETCH=2 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -1 >> gpurun_out/exp2/summary.txt
