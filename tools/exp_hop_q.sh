for r in 1 2; do for q in 1 2; do
 for K in 20 200; do
  MOMENT_HOP_Q=$q python bench.py --steps $K --warmup 5 --no-cpu-baseline --e2e-min-time 0.05 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('Q=$q K=$K', round(d['value']/1e6,2))"
 done; done; done
