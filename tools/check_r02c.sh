set -x
python -m pytest tests/test_gpu_parity.py tests/test_gpu_sharded.py tests/test_gpu_handoff.py -m gpu -x -q -p no:cacheprovider -k "not full_size" > gpurun_out/pytest_r02c.log 2>&1; tail -2 gpurun_out/pytest_r02c.log
python bench.py --steps 20 --warmup 5 > gpurun_out/bench_r02c.json 2> gpurun_out/bench_r02c.err
bash tools/bench_configs.sh r02c
