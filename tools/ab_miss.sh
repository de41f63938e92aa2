timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "extract or pipeline or worked" 2>&1 | tail -2
for C in "UK 0.18 1024" "PA 0.22 512" "PR 1.0 400"; do set -- $C
  timeout 600 python bench.py --config $1 --alpha $2 --steps 20 --warmup 3 --no-sweep --no-cpu-baseline | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); u=d['units']; print('$1', round(d['value']/1e6,3), 'extract ms', round(d['roofline']['extract_ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'miss GB/s', round(u['mean_misses']*$3/d['roofline']['extract_ms_per_step']/1e6,1))"
done
