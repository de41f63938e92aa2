# bench lines for every config at the paper's R% and at alpha=1 (+ weighted shapes), the
# same protocol as the headline (3 timed regions, median), no sweeps / CPU baseline
TAG=${1:-r02}
mkdir -p gpurun_out
for C in "PA 0.22" "PA 1.0" "TW 0.25" "TW 1.0" "UK 0.18" "UK 1.0" "PR 1.0" "PRW 1.0" "TWW 0.25" "TWW 1.0"; do
  set -- $C
  echo "== $1 alpha=$2"
  timeout 900 python bench.py --config $1 --alpha $2 --steps 40 --warmup 5 --no-sweep --no-cpu-baseline --no-pr-alpha1 2>/dev/null | tail -1
done > gpurun_out/bench_configs_$TAG.txt
