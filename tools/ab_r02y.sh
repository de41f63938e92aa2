# r02y: cold store A/B re-measured on the final build (PA at the paper's R%, UK for 1 KB rows),
# and the 2 MB-region count per batch with gid-ordered vs rank-ordered (cold store) host rows.
set -x
python tools/ab_env.py --config PA --alpha 0.22 --steps 30 --repeat 2 --variants "gid_hg25_t8:GLB_COLD_STORE=0,GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8;gid_zc:GLB_COLD_STORE=0,GLB_HOST_GATHER=0;cold_zc:GLB_COLD_STORE=1,GLB_HOST_GATHER=0;cold_hg15_t4:GLB_COLD_STORE=1,GLB_HOST_GATHER=150,GLB_HOST_GATHER_THREADS=4;cold_hg25_t8:GLB_COLD_STORE=1,GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8" > gpurun_out/cold_PA_r02y.jsonl 2>&1
python tools/ab_env.py --config UK --alpha 0.18 --steps 20 --repeat 2 --variants "gid:GLB_COLD_STORE=0;cold:GLB_COLD_STORE=1" > gpurun_out/cold_UK_r02y.jsonl 2>&1
python tools/region_count.py --config PA --alpha 0.22 --batches 5 > gpurun_out/regions_PA_r02y.jsonl 2>&1
