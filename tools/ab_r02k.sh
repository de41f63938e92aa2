set -x
for ms in 2 25 2 25; do python bench.py --steps 20 --warmup 5 --no-sweep --no-cpu-baseline --no-pr-alpha1 --clock-ms $ms | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('clock_ms', $ms, d['value'], d['runs'], d['clocks']['samples'] if d['clocks'] else None)"; done > gpurun_out/clockms_PA.txt 2>&1
