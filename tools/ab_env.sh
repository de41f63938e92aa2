# env A/B on the bench: prints value, us/step, pipelined extract us, isolated extract us + frac
run() { env "$@" timeout 900 python bench.py --no-cpu-baseline --no-sweep --steps 400 $BENCH_ARGS | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$*', '$BENCH_ARGS', round(d['value']/1e6,2), round(d['ms_per_step']*1e3,1), 'us/step; extract', round(r['extract_ms_per_step']*1e3,1), 'isolated', round(r['isolated']['extract_ms_per_step']*1e3,1), 'frac', round(r['frac'],3), round(r['isolated']['frac'],3))"; }
for i in 1 2; do
run X=0
run GLB_CACHE_ALIGN=128
run GLB_GATHER_ST=1
run GLB_CACHE_ALIGN=128 GLB_GATHER_ST=1
done
