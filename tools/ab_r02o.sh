set -x
python tools/ab_env.py --config PA --alpha 0.22 --steps 20 --repeat 3 --variants "s20:GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8" > gpurun_out/abenv20.jsonl 2>&1
python tools/ab_env.py --config PA --alpha 0.22 --steps 40 --repeat 2 --variants "s40:GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8" > gpurun_out/abenv40.jsonl 2>&1
