# L2 residency of the sampler's tables beside the pipelined gather: evict-first gather loads
# (-DGLB_GATHER_LD=1 ld.global.cs, =2 createpolicy evict_first) and the persisting-L2 window
run() { env "$@" timeout 900 python bench.py --no-cpu-baseline --no-sweep --steps 400 $BENCH_ARGS | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$*', '$BENCH_ARGS', round(d['value']/1e6,2), round(d['ms_per_step']*1e3,1), 'us/step; extract', round(r['extract_ms_per_step']*1e3,1), 'isolated', round(r['isolated']['extract_ms_per_step']*1e3,1), 'iso_step', round(r['isolated']['ms_per_step']*1e3,1))"; }
for cfg in "" "--config UK" "--config TW"; do BENCH_ARGS="$cfg"
  run GLB_LIBRARY=build/ab/libglb_WT.so
  run GLB_LIBRARY=build/ab/libglb_WT_ld1.so
  run GLB_LIBRARY=build/ab/libglb_WT_ld2.so
  run GLB_LIBRARY=build/ab/libglb_WT.so GLB_L2_PIN=1
done
