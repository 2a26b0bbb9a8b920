#!/bin/bash
# Launch-shape re-check with the indptr prefetch on (C2 bench, one knob at a time).
mkdir -p gpurun_out/sweep
run() { tag="$1"; shift; env "$@" timeout 300 python bench.py --no-cpu-baseline $EXTRA > gpurun_out/sweep/b.json 2>/dev/null;
  python -c "import json;d=json.load(open('gpurun_out/sweep/b.json'));print('$tag',round(d['value']/1e6,3),round(d['ms_per_step']*1e3,2),round(d['roofline']['frac'],3))" >> gpurun_out/sweep/summary.txt 2>&1; }
run X=0 X=0
run HOP_Q=1 MOMENT_HOP_Q=1
run HOP_Q=4 MOMENT_HOP_Q=4
run HOP_GRID=2 MOMENT_HOP_GRID=2
run COMPACT_GRID=1 MOMENT_COMPACT_GRID=1
run TMA4_BLOCKS=3 MOMENT_TMA4_BLOCKS=3
EXTRA="--inflight 12" run inflight12 X=0
EXTRA="--inflight 24" run inflight24 X=0
run X=0b X=0
