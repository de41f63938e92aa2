set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "cold_store" > gpurun_out/pytest_cold_r02g.log 2>&1; tail -2 gpurun_out/pytest_cold_r02g.log
bash tools/bench_configs.sh r02g
grep -c metric gpurun_out/bench_configs_r02g.txt
