set -x
GLB_MISS_BLOCKS=148 python tools/miss_probe.py --spans 1.0 --bins 21 --reps 3 --region-fracs 1.0,0.75,0.5,0.25,0.1 > gpurun_out/region_probe.jsonl 2>&1
