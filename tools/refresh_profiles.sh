#!/bin/bash
# Round-2 evidence refresh: GPU suite + smoke, the driver's bench commands (and the reference arm), the launch
# list of the driver command, one-step ncu of C2 and C3, warm traffic (outputs under gpurun_out/;
# copy what DESIGN.md cites into profiles/).
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.txt 2>&1
for i in 1 2; do timeout 600 python3 bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench_$i.json 2> gpurun_out/bench_$i.err; done
timeout 600 python3 bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 600 python3 bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 900 python3 bench.py --config C3 --no-cpu-baseline > gpurun_out/bench_C3.json 2> gpurun_out/bench_C3.err
timeout 600 bash tools/ncu_launches.sh gpurun_out/launches.csv C2 8 20 5 16 > gpurun_out/launch_list.txt 2>&1
timeout 900 bash tools/ncu_full.sh gpurun_out/prof_full_C2 C2 > gpurun_out/ncu_full_C2.txt 2>&1
timeout 1200 bash tools/ncu_full.sh gpurun_out/prof_full_C3 C3 > gpurun_out/ncu_full_C3.txt 2>&1
timeout 900 bash tools/ncu_warm_traffic.sh gpurun_out/warm_traffic C2 > gpurun_out/warm_traffic_C2.txt 2>&1
# (tools/sanitize.sh: compute-sanitizer was closed on the GPU pool late in round 2; profiles/r02_sanitizer_summary.txt
# is the last clean run)
rm -f gpurun_out/*.ncu-rep
