#!/bin/bash
# Results matrix (C1-C5, full size), warm per-kernel traffic and sanitizer on the current build.
mkdir -p gpurun_out
timeout 2400 python tools/results_matrix.py --out gpurun_out/results_matrix.jsonl > gpurun_out/results_matrix.txt 2>&1
timeout 600 bash tools/ncu_warm_traffic.sh gpurun_out/warm_traffic > gpurun_out/warm_traffic.txt 2>&1
timeout 900 bash tools/sanitize.sh gpurun_out/sanitize > gpurun_out/sanitize.log 2>&1
rm -f gpurun_out/*.ncu-rep
