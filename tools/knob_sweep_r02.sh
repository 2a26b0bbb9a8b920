#!/bin/bash
# Launch-shape knobs re-checked on the round-2 build: full-step us/batch at 16 lanes (tools/sampler_roofline.py)
# and the bench at K = 20, two interleaved repeats per setting. usage: tools/knob_sweep_r02.sh "K=V K2=V2 ..."
SETTINGS=${1:-"X=0 MOMENT_HOP_GRID=2 MOMENT_HOP_Q=2 MOMENT_COMPACT_GRID=1 MOMENT_COMPACT_GRID=3 MOMENT_TMA4_BLOCKS=3"}
for rep in 1 2; do
for kv in $SETTINGS; do
  s=$(env $kv python tools/sampler_roofline.py --batches 3000 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['full_step_us_per_batch'],2))")
  b=$(env $kv python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-min-time 0.05 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,2))")
  echo "$kv step_us=$s K20=$b"
done; done
