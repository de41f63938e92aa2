set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > gpurun_out/smoke_r02v.log 2>&1; tail -1 gpurun_out/smoke_r02v.log
python bench.py > gpurun_out/bench_r02v.json 2> gpurun_out/bench_r02v.err; tail -c 300 gpurun_out/bench_r02v.json
python bench.py --impl reference > gpurun_out/bench_ref_r02v.json 2> gpurun_out/bench_ref_r02v.err
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider --durations=15 > gpurun_out/pytest_gpu_r02v.log 2>&1; tail -3 gpurun_out/pytest_gpu_r02v.log
