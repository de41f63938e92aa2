# persisting-L2 window over the relabel table at pipeline depth 2: dense vs hash table, per config
python - <<'PY'
import ctypes
rt = ctypes.CDLL("libcudart.so.12")
v = ctypes.c_int()
for name, attr in [("MaxPersistingL2CacheSize", 108), ("MaxAccessPolicyWindowSize", 109), ("L2CacheSize", 38)]:
    rt.cudaDeviceGetAttribute(ctypes.byref(v), attr, 0)
    print(name, v.value)
PY
run() { env "$@" timeout 900 python bench.py --no-cpu-baseline --no-sweep --steps 400 $BENCH_ARGS | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$*', '$BENCH_ARGS', round(d['value']/1e6,2), round(d['ms_per_step']*1e3,1), 'us/step; extract', round(r['extract_ms_per_step']*1e3,1), 'isolated', round(r['isolated']['extract_ms_per_step']*1e3,1), 'iso_step', round(r['isolated']['ms_per_step']*1e3,1), d.get('relabel_table'))"; }
BENCH_ARGS=""; run GLB_L2_PIN=1; run GLB_L2_PIN=1 GLB_LIBRARY=build/ab/libglb_WT_ld1.so
BENCH_ARGS="--relabel hash"; run X=0; run GLB_L2_PIN=1
for c in UK TW PA; do
  BENCH_ARGS="--config $c --relabel hash"; run X=0; run GLB_L2_PIN=1
done
