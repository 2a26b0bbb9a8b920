#!/bin/bash
# Lanes in flight vs seeds/s at the driver's K (bench.py --steps K): one JSON summary line per setting.
# usage: tools/sweep_inflight.sh K "4 8 10 12 16 20" [extra bench args]
K=$1; shift; PS=$1; shift
for P in $PS; do
  python bench.py --steps $K --warmup 5 --inflight $P --no-cpu-baseline --e2e-min-time 0.05 "$@" 2>/dev/null |
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({'K': $K, 'P': $P, 'Mseeds': d['value']/1e6, 'us_step': d['ms_per_step']*1e3, 'region_ms': d['config']['region_ms']}))"
done
