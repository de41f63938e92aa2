set -x
for T in memcheck racecheck synccheck; do echo "== $T"; timeout 1200 compute-sanitizer --tool $T --print-limit 20 python tools/sanitize.py 2>&1 | tail -6; done > gpurun_out/sanitizer_r02.txt 2>&1
python -m pytest tests/test_gpu_parity.py tests/test_gpu_handoff.py tests/test_gpu_sharded.py -m gpu -x -q -p no:cacheprovider -k "not full_size" > gpurun_out/pytest_parity_r02b.log 2>&1
bash tools/bench_configs.sh r02b
