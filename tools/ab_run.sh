# A/B of library builds on the bench config: [BENCH_ARGS="--config UK"] [RUNS=2] bash tools/ab_run.sh lib1.so lib2.so ...
for L in "$@"; do for i in $(seq ${RUNS:-2}); do
  GLB_LIBRARY=$L timeout 900 python bench.py --no-cpu-baseline --no-sweep --steps ${STEPS:-400} $BENCH_ARGS | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$L', '$BENCH_ARGS', round(d['value']/1e6,2), round(d['ms_per_step']*1e3,1), 'us/step extract', round(d['roofline']['extract_ms_per_step']*1e3,1), d['gpu_launches'])"
done; done
