#!/bin/bash
# Warm-cache DRAM traffic per kernel of one C2 step (ncu --cache-control none: caches NOT flushed between
# launches, so each kernel sees the L2 state the previous kernels left).
OUT=${1:-gpurun_out/warm_traffic}
ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_write.sum,lts__t_sectors_srcunit_tex_op_red.sum \
  -k "regex:hop_|bitscan|compact|init_kernel|gather_" -s 24 -c 24 --csv --log-file "$OUT.csv" \
  python bench.py --config ${2:-C2} --steps 4 --warmup 3 --inflight 1 --no-cpu-baseline --min-time 0 --e2e-min-time 0 > /dev/null 2>&1
python - "$OUT.csv" <<'PY'
import csv, sys
from collections import defaultdict
rows = [r for r in csv.DictReader(l for l in open(sys.argv[1]) if l.startswith('"'))]
agg = defaultdict(lambda: defaultdict(float)); cnt = defaultdict(set)
for r in rows:
    k = r["Kernel Name"].replace("(anonymous namespace)::", "").replace("moment::", "").replace("void ", "").split("(")[0][:32]
    v = float(r["Metric Value"].replace(",", ""))
    u = r["Metric Unit"]
    if u in ("Kbyte",): v *= 1e3
    if u in ("Mbyte",): v *= 1e6
    if u in ("Gbyte",): v *= 1e9
    if u in ("usecond",): v *= 1e3
    if u in ("msecond",): v *= 1e6
    agg[k][r["Metric Name"]] += v; cnt[k].add(r["ID"])
steps = 3
print(f"{'kernel':32s} {'us':>7s} {'dram_rd_MB':>10s} {'dram_wr_MB':>10s} {'l2_rd_sect_M':>12s} {'l2_wr_M':>8s} {'l2_red_M':>8s}")
tot = defaultdict(float)
for k, m in agg.items():
    vals = [m["gpu__time_duration.sum"] / steps / 1e3, m["dram__bytes_read.sum"] / steps / 1e6, m["dram__bytes_write.sum"] / steps / 1e6,
            m["lts__t_sectors_srcunit_tex_op_read.sum"] / steps / 1e6, m["lts__t_sectors_srcunit_tex_op_write.sum"] / steps / 1e6,
            m["lts__t_sectors_srcunit_tex_op_red.sum"] / steps / 1e6]
    for i, v in enumerate(vals): tot[i] += v
    print(f"{k:32s} " + " ".join(f"{v:10.2f}" for v in vals))
print(f"{'total per step':32s} " + " ".join(f"{tot[i]:10.2f}" for i in range(6)))
PY
