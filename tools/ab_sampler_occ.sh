# sampler occupancy next to the pipelined gather: sampler grid blocks/SM x compaction register cap
run() { env "$@" timeout 900 python bench.py --no-cpu-baseline --no-sweep --steps 400 $BENCH_ARGS | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$*', '$BENCH_ARGS', round(d['value']/1e6,2), round(d['ms_per_step']*1e3,1), 'us/step; extract', round(r['extract_ms_per_step']*1e3,1), 'isolated', round(r['isolated']['extract_ms_per_step']*1e3,1), 'iso_step', round(r['isolated']['ms_per_step']*1e3,1))"; }
for L in build/ab/libglb_WT.so build/ab/libglb_WT_c4.so build/ab/libglb_WT_c2.so; do
  for B in 8 6 4 12; do run GLB_LIBRARY=$L GLB_SAMPLE_BPS=$B; done
done
