# r02p2: host part chunk count with the cold store (PA, paper R%), 3 rounds
set -x
B="GLB_COLD_STORE=1,GLB_HOST_GATHER_THREADS=4"
V="def:$B,GLB_HOST_GATHER=150"
V="$V;ch2:$B,GLB_HOST_GATHER=150,GLB_HOST_GATHER_CHUNKS=2"
V="$V;ch1:$B,GLB_HOST_GATHER=150,GLB_HOST_GATHER_CHUNKS=1"
V="$V;ch2f20:$B,GLB_HOST_GATHER=200,GLB_HOST_GATHER_CHUNKS=2"
V="$V;ch2f10:$B,GLB_HOST_GATHER=100,GLB_HOST_GATHER_CHUNKS=2"
V="$V;ch2t6:GLB_COLD_STORE=1,GLB_HOST_GATHER_THREADS=6,GLB_HOST_GATHER=150,GLB_HOST_GATHER_CHUNKS=2"
python tools/ab_env.py --config PA --alpha 0.22 --steps 40 --repeat 3 --variants "$V" > gpurun_out/chunks_PA_r02p2.jsonl 2>&1
