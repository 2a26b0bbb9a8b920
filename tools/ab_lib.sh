for i in 1 2; do
for lib in libmoment_old.so libmoment.so; do
MOMENT_LIB_PATH=$PWD/paper_conf_sc_shi0s0x0w25_b200/lib/$lib python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-min-time 0.05 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$lib', round(d['value']/1e6,2), round(r['launch_ms']*1e3,2), round(r['frac'],3), round(r['concurrent']['frac'],3))"
done; done
