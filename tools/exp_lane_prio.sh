#!/bin/bash
# Lane stream priorities at the driver's K = 20 (MOMENT_LANE_PRIO: half | hi:N = the first N lanes high), with
# the lanes in flight (--inflight P): the K mod P lanes that run one more batch than the rest, high.
for r in 1 2; do for pm in "16 half" "16 hi:4" "12 hi:8" "14 hi:6" "18 hi:2" "20 half" "10 half"; do
  set -- $pm
  MOMENT_LANE_PRIO=$2 python bench.py --steps 20 --warmup 5 --inflight $1 --no-cpu-baseline --e2e-min-time 0.05 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('P=$1 $2 K=20', round(d['value']/1e6,2))"
done; done
