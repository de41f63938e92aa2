set -x
python bench.py > gpurun_out/bench_default_r02.json 2> gpurun_out/bench_default_r02.err
bash tools/bench_configs.sh r02
ncu --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv --log-file gpurun_out/launches_r02.csv \
    python bench.py --steps 4 --warmup 3 --runs 1 --no-sweep --no-cpu-baseline --no-pr-alpha1 > gpurun_out/launches_r02.log 2>&1
