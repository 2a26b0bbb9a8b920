#!/bin/bash
# One `ncu --set full` capture of every product kernel of one warm bench step (1 lane, C2 by default).
OUT=${1:-gpurun_out/prof_full}
CFG=${2:-C2}
KRE="regex:hop_|bitscan|compact|init_kernel|gather_"
ncu --set full --clock-control none --import-source on -k "$KRE" -s 24 -c 8 -o "$OUT" \
    python bench.py --config "$CFG" --steps 2 --warmup 3 --inflight 1 --no-cpu-baseline --min-time 0 --e2e-min-time 0 > /dev/null 2>&1
ncu -i "$OUT.ncu-rep" --page raw --csv \
    --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,launch__grid_size,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,lts__t_bytes.sum,smsp__average_warp_latency_issue_stalled_long_scoreboard,sm__throughput.avg.pct_of_peak_sustained_elapsed \
    > "$OUT.csv" 2>&1
python tools/summarize_ncu.py "$OUT.csv"
