set -x
for i in 1 2 3 4; do GLB_HG_STATS=1 python bench.py --steps 20 --warmup 5 --no-sweep --no-cpu-baseline --no-pr-alpha1 > gpurun_out/var_$i.json 2> gpurun_out/var_$i.err; done
