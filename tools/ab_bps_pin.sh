# gather blocks/SM on the extract stream, with the relabel table pinned (PR, PRW)
run() { env "$@" timeout 900 python bench.py --no-cpu-baseline --no-sweep --k-sweep "" --steps 400 $BENCH_ARGS | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$*', '$BENCH_ARGS', round(d['value']/1e6,2), round(d['ms_per_step']*1e3,1), 'us/step; extract', round(r['extract_ms_per_step']*1e3,1), 'isolated', round(r['isolated']['extract_ms_per_step']*1e3,1))"; }
for cfg in "" "--config PRW"; do BENCH_ARGS="$cfg"
for B in 2 3 4; do run GLB_GATHER_BPS_PIPE=$B; done; done
