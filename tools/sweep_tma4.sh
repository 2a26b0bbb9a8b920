#!/bin/bash
# tile::gather4 blocks per SM (MOMENT_TMA4_BLOCKS) vs the bench value and the gather's single-launch roofline
for b in ${1:-1 2 3 4}; do
  MOMENT_TMA4_BLOCKS=$b python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-min-time 0.05 2>/dev/null |
    python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('blocks/SM $b', round(d['value']/1e6,2), 'M seeds/s; gather', round(r['launch_ms']*1e3,2), 'us frac', round(r['frac'],3), 'b2b', round(r['back_to_back']['frac'],3), 'conc', round(r['concurrent']['frac'],3))"
done
