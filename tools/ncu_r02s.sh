# r02s: ncu --set full of the PA sampler kernels (k_rwalk, k_compact; the headline's sampling half),
# one launch each at the last hop of a step (cold store and host part off: ncu OOM, r02d)
set -x
B="python bench.py --steps 4 --warmup 3 --runs 1 --no-sweep --no-cpu-baseline --no-pr-alpha1 --pipeline 1 --cold-store off --host-gather 0"
for K in k_rwalk k_compact; do
  ncu --set full --clock-control none --cache-control none --import-source on -k regex:$K -s 470 -c 3 \
      -o gpurun_out/prof_${K}_PA_r02s $B > gpurun_out/ncu_${K}_PA_r02s.log 2>&1; echo "$K rc=$?"
done
