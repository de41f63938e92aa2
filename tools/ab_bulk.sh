# bulk (TMA) hit gather vs LSU gather, pipelined bench (PR and UK), smem budget sweep
run() { env "$@" timeout 900 python bench.py --no-cpu-baseline --no-sweep --steps 400 $BENCH_ARGS | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$*', '$BENCH_ARGS', round(d['value']/1e6,2), round(d['ms_per_step']*1e3,1), 'us/step; extract', round(r['extract_ms_per_step']*1e3,1), 'isolated', round(r['isolated']['extract_ms_per_step']*1e3,1), 'iso_step', round(r['isolated']['ms_per_step']*1e3,1))"; }
for cfg in "" "--config UK"; do
BENCH_ARGS="$cfg"
run GLB_GATHER_BULK=0
run GLB_GATHER_BULK=1
run GLB_GATHER_BULK=1 GLB_GATHER_BULK_SMEM=65536
run GLB_GATHER_BULK=1 GLB_GATHER_BULK_SMEM=131072
run GLB_GATHER_BULK=1 GLB_GATHER_BPS_PIPE=3
done
