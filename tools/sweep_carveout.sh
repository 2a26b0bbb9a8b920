#!/bin/bash
# Shared-memory carveout preferences (percent of the unified L1/shared storage given to shared memory) for the
# sampler kernels and the gather kernels separately: bench K=20 (value, gather roofline) and K=200, 2 repeats.
for rep in 1 2; do DEF="X=0 MOMENT_CARVEOUT=25 MOMENT_CARVEOUT_SAMPLE=0 MOMENT_CARVEOUT_SAMPLE=25 MOMENT_CARVEOUT_SAMPLE=10"
 for kv in ${1:-$DEF}; do
 a=$(env $kv python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-min-time 0.05 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,2), round(d['roofline']['frac'],3))")
 b=$(env $kv python bench.py --steps 200 --warmup 5 --no-cpu-baseline --e2e-min-time 0.05 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,2))")
 echo "$kv K20=$a K200=$b"
done; done
