#!/bin/bash
# Launch list of a short bench run (cold-cache, serialised per-launch times; compare SHARES only).
OUT=${1:-gpurun_out/launches.csv}
CFG=${2:-C2}
ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:hop_|bitscan|compact|init_kernel|gather_|bucket_|queue_|relay_|hotness" -c 300 --csv --log-file "$OUT" \
    python bench.py --config "$CFG" --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1 || true
python tools/summarize_launches.py "$OUT"
