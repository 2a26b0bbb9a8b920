#!/bin/bash
# Round-2 evidence refresh: the driver's bench command, its launch list, one-step ncu of C2 and C3, warm traffic,
# sanitizers (outputs under gpurun_out/; copy what DESIGN.md cites into profiles/).
set -x
mkdir -p gpurun_out
python3 bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/r02_bench_C2.json 2> gpurun_out/r02_bench_C2.err
bash tools/ncu_launches.sh gpurun_out/r02_launch_list_C2.csv C2 8 20 5 16 > gpurun_out/r02_launch_list_C2.txt 2>&1
bash tools/ncu_full.sh gpurun_out/r02_prof_full_C2 C2 > gpurun_out/r02_ncu_set_full_one_step_C2.txt 2>&1
bash tools/ncu_full.sh gpurun_out/r02_prof_full_C3 C3 > gpurun_out/r02_ncu_set_full_one_step_C3.txt 2>&1
bash tools/ncu_warm_traffic.sh gpurun_out/r02_warm_traffic C2 > gpurun_out/r02_warm_traffic_C2.txt 2>&1
bash tools/sanitize.sh gpurun_out/sanitize_r02 > /dev/null 2>&1
