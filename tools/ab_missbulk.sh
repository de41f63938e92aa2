# host misses: LSU zero-copy gather vs one cp.async.bulk per row (GLB_MISS_BULK=1), paper R% configs
run() { env "$@" timeout 900 python bench.py --no-cpu-baseline --no-sweep --k-sweep "" --steps 60 $BENCH_ARGS | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); r=d['roofline']; u=d['units']; print('$*', '$BENCH_ARGS', round(d['value']/1e6,3), round(d['ms_per_step'],3), 'ms/step; extract', round(r['extract_ms_per_step'],3), 'ms; misses/step', round(u['mean_misses']), 'host GB/s', round(u['mean_misses']*d['config']['feat_dim']*4/(r['extract_ms_per_step']*1e-3)/1e9,1))"; }
for c in "TW --alpha 0.25" "UK --alpha 0.18" "PA --alpha 0.22"; do BENCH_ARGS="--config $c"
  run X=0; run GLB_MISS_BULK=1; run GLB_MISS_BULK=1 GLB_GATHER_BULK_SMEM=65536; run GLB_MISS_BULK=1 GLB_GATHER_BULK_SMEM=196608
done
