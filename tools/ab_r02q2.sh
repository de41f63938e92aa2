# r02q2: host share 0.10 vs 0.15 and 2 vs 4 chunks with the cold store (PA, paper R%), 3 rounds
set -x
B="GLB_COLD_STORE=1,GLB_HOST_GATHER_THREADS=4"
V="def:$B,GLB_HOST_GATHER=150"
V="$V;ch2f10:$B,GLB_HOST_GATHER=100,GLB_HOST_GATHER_CHUNKS=2"
V="$V;f10:$B,GLB_HOST_GATHER=100"
V="$V;ch2f10t3:GLB_COLD_STORE=1,GLB_HOST_GATHER_THREADS=3,GLB_HOST_GATHER=100,GLB_HOST_GATHER_CHUNKS=2"
V="$V;ch2f12:$B,GLB_HOST_GATHER=120,GLB_HOST_GATHER_CHUNKS=2"
python tools/ab_env.py --config PA --alpha 0.22 --steps 40 --repeat 3 --variants "$V" > gpurun_out/share_PA_r02q2.jsonl 2>&1
