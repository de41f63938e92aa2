set -x
python bench.py > gpurun_out/bench_r02l.json 2> gpurun_out/bench_r02l.err; tail -c 1500 gpurun_out/bench_r02l.json
