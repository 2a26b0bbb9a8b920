set -x
mkdir -p gpurun_out
python bench.py > gpurun_out/bench3.json 2> gpurun_out/bench3.err
bash tools/ncu_launches.sh gpurun_out/launches.csv C2 8 > gpurun_out/launch_list.txt 2>&1
bash tools/ncu_full.sh gpurun_out/prof_full_C3 C3 > gpurun_out/ncu_full_C3.txt 2>&1
bash tools/ncu_warm_traffic.sh gpurun_out/warm_traffic > gpurun_out/warm_traffic.txt 2>&1
bash tools/sanitize.sh gpurun_out/sanitize2 > /dev/null 2>&1
