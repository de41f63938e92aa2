# Round profile capture on the bench configuration (1 GPU):
#   1. ncu launch list (every launch's gpu__time_duration, no cache flush)
#   2. ncu --set full of the top kernels (k_gather, k_compact, k_khop)
# usage: bash tools/prof.sh <tag>   -> gpurun_out/*_<tag>.*
set -x
TAG=${1:-r01}
B="python bench.py --steps 10 --warmup 3 --no-sweep --no-cpu-baseline"
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -c 2000 --csv --log-file gpurun_out/launches_$TAG.csv $B > gpurun_out/b_ncu_$TAG.log 2>&1
[ "$2" = "launches" ] && exit 0
for K in k_gather k_compact k_khop k_seed_init k_fixup; do
  ncu --set full --clock-control none --cache-control none --import-source on -k regex:$K -s 6 -c 2 -o gpurun_out/prof_${K}_$TAG $B > /dev/null 2>&1
done
ls -la gpurun_out
