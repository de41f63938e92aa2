# A/B of library builds on the bench config: bash tools/ab_run.sh lib1.so lib2.so ...
for L in "$@"; do for i in 1 2; do
  GLB_LIBRARY=$L timeout 600 python bench.py --no-cpu-baseline --no-sweep "${BENCH_ARGS[@]}" | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$L', round(d['value']/1e6,2), round(d['ms_per_step']*1e3,1), 'us/step extract', round(d['roofline']['extract_ms_per_step']*1e3,1), d['gpu_launches'])"
done; done
