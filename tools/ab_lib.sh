#!/bin/bash
# A/B of two builds of libmoment.so on one box (MOMENT_LIB_PATH): bench value at K = 20 and the gather's single
# launch, then the sampling-only / full-step throughput, alternating ${REPS:-2} times.
# usage: tools/ab_lib.sh [old.so] [new.so]   (old default: paper_conf_sc_shi0s0x0w25_b200/lib/libmoment_old.so)
A=${1:-$PWD/paper_conf_sc_shi0s0x0w25_b200/lib/libmoment_old.so}
B=${2:-$PWD/paper_conf_sc_shi0s0x0w25_b200/lib/libmoment.so}
for i in $(seq ${REPS:-2}); do
for lib in $A $B; do
MOMENT_LIB_PATH=$lib python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-min-time 0.05 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$(basename $lib)', 'K=20', round(d['value']/1e6,2), 'gather us', round(r['launch_ms']*1e3,2), 'frac', round(r['frac'],3))"
MOMENT_LIB_PATH=$lib python tools/sampler_roofline.py --batches 3000 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$(basename $lib)', 'sampling', round(d['sampling_only_us_per_batch'],2), 'step', round(d['full_step_us_per_batch'],2))"
done; done
