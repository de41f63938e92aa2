# hits gathered in lid order (GLB_GATHER_LIDORDER=1) vs from the hit list
set -x
python -m pytest tests/test_gpu_parity.py tests/test_gpu_sharded.py -m gpu -x -q -p no:cacheprovider -k "extract or sharded_extract_sample" > gpurun_out/pytest_lidorder.log 2>&1; tail -2 gpurun_out/pytest_lidorder.log
python tools/ab_env.py --config PR --alpha 1.0 --steps 200 --repeat 2 --variants "base:;lid:GLB_GATHER_LIDORDER=1" > gpurun_out/lid_PR.jsonl 2>&1
python tools/ab_env.py --config UK --alpha 1.0 --steps 60 --repeat 2 --variants "base:;lid:GLB_GATHER_LIDORDER=1" > gpurun_out/lid_UK.jsonl 2>&1
python tools/ab_env.py --config TW --alpha 1.0 --steps 60 --repeat 2 --variants "base:;lid:GLB_GATHER_LIDORDER=1" > gpurun_out/lid_TW.jsonl 2>&1
python tools/ab_env.py --config PA --alpha 1.0 --steps 60 --repeat 2 --variants "base:;lid:GLB_GATHER_LIDORDER=1" > gpurun_out/lid_PA1.jsonl 2>&1
python tools/ab_env.py --config PA --alpha 0.22 --steps 30 --repeat 2 --variants "base:GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8;lid:GLB_GATHER_LIDORDER=1,GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8" > gpurun_out/lid_PA.jsonl 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for V in 0 1; do
  GLB_GATHER_LIDORDER=$V ncu --metrics $M --clock-control none --cache-control none -k "regex:k_gather" -s 4 -c 3 --csv \
      --log-file gpurun_out/lid_ncu_PR_$V.csv python bench.py --config PR --steps 4 --warmup 3 --runs 1 --no-sweep --no-cpu-baseline --pipeline 1 --no-pr-alpha1 > /dev/null 2>&1
done
