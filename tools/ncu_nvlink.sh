#!/bin/bash
# NVLink and PCIe bytes of the partitioned / tiered gathers on a multi-GPU box ("NVLink rx/tx bytes,
# PCIe read bytes" per representative batch). Profiles rank 0's gather and relay kernels of a short partitioned
# bench run under torchrun; the other ranks run unprofiled (ncu attaches to rank 0 only through the wrapper).
# Needs >= 2 GPUs (one process per GPU); on this pool's one-GPU boxes peer pointers are same-device IPC mappings
# and these counters read 0.
#   usage: tools/ncu_nvlink.sh [N] [C3|C4] [ddak-rep|ddak-tiered] [out]
N=${1:-2}; CFG=${2:-C3}; PL=${3:-ddak-rep}; OUT=${4:-gpurun_out/ncu_nvlink}
METRICS=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,nvlrx__bytes_data_user.sum,nvltx__bytes_data_user.sum,pcie__read_bytes.sum,pcie__write_bytes.sum
cat > /tmp/ncu_rank0.sh <<EOS
#!/bin/bash
if [ "\$RANK" = "0" ]; then
  exec ncu --metrics $METRICS --clock-control none -k "regex:gather|relay" -s 64 -c 16 --csv --log-file $OUT.csv python "\$@"
else
  exec python "\$@"
fi
EOS
chmod +x /tmp/ncu_rank0.sh
python -m torch.distributed.run --nnodes=1 --nproc-per-node=$N --master-addr=127.0.0.1 --master-port=29533 \
    --no-python /tmp/ncu_rank0.sh bench.py --gpus $N --config $CFG --placement $PL --steps 20 --warmup 3 \
    --inflight 4 --min-time 0.2 --e2e-min-time 0.05 --no-cpu-baseline > $OUT.log 2>&1
python - "$OUT.csv" <<'PY'
import csv, sys
from collections import defaultdict
rows = [r for r in csv.DictReader(l for l in open(sys.argv[1]) if l.startswith('"'))]
agg = defaultdict(lambda: defaultdict(float)); n = defaultdict(set)
for r in rows:
    k = r["Kernel Name"].split("(")[0][-40:]
    u = r["Metric Unit"]; v = float(r["Metric Value"].replace(",", ""))
    v *= {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "usecond": 1e3, "msecond": 1e6}.get(u, 1)
    agg[k][r["Metric Name"]] += v; n[k].add(r["ID"])
for k, m in agg.items():
    c = len(n[k]); t = m["gpu__time_duration.sum"] / c
    nv = (m["nvlrx__bytes_data_user.sum"] + m["nvltx__bytes_data_user.sum"]) / c
    print(f"{k:40s} launches {c:3d}  {t / 1e3:8.1f} us  nvl rx {m['nvlrx__bytes_data_user.sum'] / c / 1e6:8.2f} MB"
          f"  tx {m['nvltx__bytes_data_user.sum'] / c / 1e6:8.2f} MB  ({nv / t:6.1f} GB/s)  pcie rd "
          f"{m['pcie__read_bytes.sum'] / c / 1e6:8.2f} MB  dram rd {m['dram__bytes_read.sum'] / c / 1e6:8.2f} MB")
PY
