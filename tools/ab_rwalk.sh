# random-walk sampler register cap (-DGLB_RWALK_MINB) on PA, pipelined and isolated
run() { env "$@" timeout 900 python bench.py --no-cpu-baseline --no-sweep --k-sweep "" --steps 200 $BENCH_ARGS | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$*', '$BENCH_ARGS', round(d['value']/1e6,2), round(d['ms_per_step']*1e3,1), 'us/step; extract', round(r['extract_ms_per_step']*1e3,1), 'iso_step', round(r['isolated']['ms_per_step']*1e3,1))"; }
BENCH_ARGS="--config PA"
for L in build/ab/libglb_WT.so build/ab/libglb_WT_rw6.so build/ab/libglb_WT_rw8.so; do run GLB_LIBRARY=$L; done
