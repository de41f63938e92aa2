set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > gpurun_out/smoke_r02c.log 2>&1; tail -1 gpurun_out/smoke_r02c.log
python bench.py > gpurun_out/bench_r02c.json 2> gpurun_out/bench_r02c.err; tail -c 600 gpurun_out/bench_r02c.json
python bench.py --impl reference > gpurun_out/bench_ref_r02c.json 2> gpurun_out/bench_ref_r02c.err
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider --durations=15 > gpurun_out/pytest_gpu_r02c.log 2>&1; tail -3 gpurun_out/pytest_gpu_r02c.log
