#!/bin/bash
# ncu --set full of ONE kernel (regex $1) of a warm C2 step; prints warp-stall and memory summary.
KRE=$1; OUT=${2:-gpurun_out/prof_kernel}; SKIP=${3:-3}
ncu --set full --clock-control none --import-source on -k "regex:$KRE" -s "$SKIP" -c 1 -o "$OUT" \
    python bench.py --config C2 --steps 2 --warmup 3 --inflight 1 --no-cpu-baseline --min-time 0 --e2e-min-time 0 > /dev/null 2>&1
ncu -i "$OUT.ncu-rep" --page details --csv 2>/dev/null | python tools/ncu_details.py
