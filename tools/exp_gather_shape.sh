#!/bin/bash
# gather4 launch shapes (tile rows x blocks per SM: MOMENT_TMA4_ROWS, MOMENT_TMA4_BLOCKS) in the step and alone:
# full step at 16 lanes (tools/exp_variants.py) and the bench at K = 20 (value + the single-launch roofline), two
# repeats. (The stage-count / store-lag rows of profiles/r02_sampler_experiments.txt came from experiment builds.)
S=${SHAPES:-"- MOMENT_TMA4_ROWS=32,MOMENT_TMA4_BLOCKS=2 MOMENT_TMA4_ROWS=16,MOMENT_TMA4_BLOCKS=2 MOMENT_TMA4_ROWS=8,MOMENT_TMA4_BLOCKS=6"}
python tools/exp_variants.py --config C2 --lanes 16 $S
for r in 1 2; do for kv in $S; do
  e=""; [ "$kv" != "-" ] && e=$(echo $kv | tr ',' ' ')
  env $e python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-min-time 0.05 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$kv', 'K=20', round(d['value']/1e6,2), 'gather us', round(r['launch_ms']*1e3,2), 'frac', round(r['frac'],3), 'concurrent', round(r['concurrent']['frac'],3))"
done; done
