set -x
python bench.py --steps 20 --warmup 5 > gpurun_out/bench_r02e.json 2> gpurun_out/bench_r02e.err
python -m pytest tests/test_gpu_fullsize.py -m gpu -x -q -p no:cacheprovider -k "pa_fullsize" > gpurun_out/pytest_pa_cold.log 2>&1; tail -2 gpurun_out/pytest_pa_cold.log
