#!/bin/bash
# A/B of several builds of libmoment.so (MOMENT_LIB_PATH), interleaved ${REPS:-2} times: bench value at K = 20
# (16 lanes) and the full-step / sampling-only us per batch at 16 lanes (tools/sampler_roofline.py).
# usage: tools/ab_multi.sh a.so b.so ...
for i in $(seq ${REPS:-2}); do
for lib in "$@"; do
  b=$(MOMENT_LIB_PATH=$lib python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-min-time 0.05 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,2), 'gather', round(d['roofline']['frac'],3))")
  s=$(MOMENT_LIB_PATH=$lib python tools/sampler_roofline.py --batches 3000 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sampling', round(d['sampling_only_us_per_batch'],2), 'step', round(d['full_step_us_per_batch'],2))")
  echo "$(basename $lib) K=20 $b $s"
done; done
