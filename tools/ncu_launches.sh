#!/bin/bash
# Launch list of the FIRST TIMED REGION of the driver's bench command (python bench.py --steps K --warmup W,
# P lanes): cold-cache, serialised per-launch times (ncu --clock-control none); compare SHARES only.
# L = product kernels per step matched by the regex (C2: 3 hop samplers, 3 bitscans, compact, gather = 8;
# set_call is not matched); the W x P warm-up steps are skipped, the K steps of the first region captured.
OUT=${1:-gpurun_out/launches.csv}
CFG=${2:-C2}
L=${3:-8}
K=${4:-20}
W=${5:-5}
P=${6:-16}
ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:hop_|bitscan|compact|init_kernel|gather_" \
    -s $((W * P * L)) -c $((K * L)) --csv --log-file "$OUT" \
    python bench.py --config "$CFG" --gpus 1 --steps $K --warmup $W --inflight $P --no-cpu-baseline --min-time 0 \
    --e2e-min-time 0 > /dev/null 2>&1 || true
python tools/summarize_launches.py "$OUT"
