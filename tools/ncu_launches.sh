#!/bin/bash
# Launch list of a short bench run (cold-cache, serialised per-launch times; compare SHARES only).
set -e
OUT=${1:-gpurun_out/launches.csv}
ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file "$OUT" \
    python bench.py --steps 6 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1 || true
python tools/summarize_launches.py "$OUT"
