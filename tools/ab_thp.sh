for A in cuda register; do
  timeout 900 python bench.py --config PA --alpha 0.22 --steps 20 --warmup 3 --no-sweep --no-cpu-baseline --host-alloc $A | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); u=d['units']; print('PA alloc=$A', round(d['value']/1e6,3), 'extract ms', round(d['roofline']['extract_ms_per_step'],3), 'misses', u['mean_misses'], 'GB/s', round(u['mean_misses']*512/d['roofline']['extract_ms_per_step']/1e6,1), d['preprocess_s'])"
done
