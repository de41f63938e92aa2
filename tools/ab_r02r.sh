set -x
python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "extract" > gpurun_out/pytest_mfirst.log 2>&1; tail -2 gpurun_out/pytest_mfirst.log
python tools/ab_env.py --config PA --alpha 0.22 --steps 30 --repeat 3 --depths 2,1 --variants "base:GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8;first:GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8,GLB_MISSES_FIRST=1;first_zc:GLB_HOST_GATHER=0,GLB_MISSES_FIRST=1,GLB_MISS_BLOCKS=148" > gpurun_out/mfirst_PA.jsonl 2>&1
python tools/ab_env.py --config UK --alpha 0.18 --steps 20 --repeat 2 --variants "base:;mb148:GLB_MISS_BLOCKS=148;first148:GLB_MISS_BLOCKS=148,GLB_MISSES_FIRST=1;first200:GLB_MISS_BLOCKS=200,GLB_MISSES_FIRST=1" > gpurun_out/mfirst_UK.jsonl 2>&1
python tools/ab_env.py --config TW --alpha 0.25 --steps 20 --repeat 2 --variants "base:;first148:GLB_MISS_BLOCKS=148,GLB_MISSES_FIRST=1" > gpurun_out/mfirst_TW.jsonl 2>&1
