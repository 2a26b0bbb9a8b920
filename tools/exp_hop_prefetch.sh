mkdir -p gpurun_out/exp
for cfg in C2 C3; do for r in 1 2; do for p in 0 1; do
  MOMENT_HOP_PREFETCH=$p timeout 300 python bench.py --config $cfg --no-cpu-baseline > gpurun_out/exp/b_${cfg}_p${p}_$r.json 2>gpurun_out/exp/err_${cfg}_p${p}_$r.txt
  python -c "import json;d=json.load(open('gpurun_out/exp/b_${cfg}_p${p}_$r.json'));print('$cfg p=$p r=$r',round(d['value']/1e6,3),round(d['ms_per_step']*1e3,2),round(d['roofline']['frac'],3))" >> gpurun_out/exp/summary.txt 2>&1
done; done; done
MOMENT_HOP_PREFETCH=1 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/exp/parity_p1.txt 2>&1
