set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_r02.log 2>&1
python bench.py --steps 20 --warmup 5 > gpurun_out/bench_final_r02.json 2> gpurun_out/bench_final_r02.err
python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/bench_ref_r02.json 2> gpurun_out/bench_ref_r02.err
python -m pytest tests -m gpu -x -q -p no:cacheprovider --durations=15 > gpurun_out/pytest_gpu_final.log 2>&1
