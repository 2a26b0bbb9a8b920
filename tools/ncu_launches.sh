#!/bin/bash
# Launch list of the TIMED steps of a short bench run (cold-cache, serialised per-launch times; compare
# SHARES only). L = product kernels per step matched by the regex (C2: 3 hop samplers, 3 bitscans, compact,
# gather = 8; set_call is not matched); the W warm-up steps are skipped, the K timed steps captured.
OUT=${1:-gpurun_out/launches.csv}
CFG=${2:-C2}
L=${3:-8}
W=3
K=10
ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:hop_|bitscan|compact|init_kernel|gather_" \
    -s $((W * L)) -c $((K * L)) --csv --log-file "$OUT" \
    python bench.py --config "$CFG" --steps $K --warmup $W --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1 || true
python tools/summarize_launches.py "$OUT"
