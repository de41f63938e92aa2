set -x
python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "extract" > gpurun_out/pytest_extract.log 2>&1; tail -3 gpurun_out/pytest_extract.log
for W in 0 1; do GLB_GATHER_WARP=$W python tools/miss_probe.py --spans 1.0,0.25 --bins 21 > gpurun_out/miss_probe_w$W.jsonl 2>&1; done
for W in 0 1; do GLB_GATHER_WARP=$W python bench.py --config PR --alpha 1.0 --no-sweep --no-cpu-baseline --steps 100 --runs 3 > gpurun_out/bench_PR_w$W.json 2> gpurun_out/bench_PR_w$W.err; done
python tools/miss_ab.py --config PA --alpha 0.22 --bins 21 --env GLB_GATHER_WARP=1 > gpurun_out/miss_ab_PA_w1.jsonl 2>&1
