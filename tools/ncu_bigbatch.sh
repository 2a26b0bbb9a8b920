#!/bin/bash
# ncu --set full of the sampling kernels of ONE warm big-batch step (B seeds, sample only, 1 lane):
# where a large hop kernel spends its time. 3 warm-up steps x 7 kernels are skipped.
B=${1:-16384}; OUT=${2:-gpurun_out/prof_big}
ncu --set full --clock-control none --import-source on -k "regex:hop_|bitscan|compact" -s 21 -c 7 -o "$OUT" \
    python tools/exp_bigbatch.py --sizes $B --steps 1 > /dev/null 2>&1
ncu -i "$OUT.ncu-rep" --page details --csv 2>/dev/null | python tools/ncu_details.py
