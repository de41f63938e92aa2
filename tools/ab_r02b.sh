# r02: block smem-staged relabel pre-dedup (GLB_RELABEL_DEDUP=2) vs warp (1) vs none, and
# host-gather tuning on PA (gather blocks/SM on the extract stream, scatter grid, share)
set -x
python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "fanout_variants or tiny_every" > gpurun_out/pytest_dedup2.log 2>&1; tail -2 gpurun_out/pytest_dedup2.log
python tools/ab_env.py --config TW --alpha 1.0 --steps 60 --repeat 2 --variants "base:;dedup1:GLB_RELABEL_DEDUP=1;dedup2:GLB_RELABEL_DEDUP=2" > gpurun_out/dedup2_TW.jsonl 2>&1
python tools/ab_env.py --config UK --alpha 1.0 --steps 60 --repeat 2 --variants "base:;dedup2:GLB_RELABEL_DEDUP=2" > gpurun_out/dedup2_UK.jsonl 2>&1
python tools/ab_env.py --config PR --alpha 1.0 --steps 200 --repeat 2 --variants "base:;dedup2:GLB_RELABEL_DEDUP=2" > gpurun_out/dedup2_PR.jsonl 2>&1
V="base:GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8"
for f in 250 300 350; do for b in 1 2; do for sb in 0 32; do
  V="$V;f${f}_bps${b}_sb${sb}:GLB_HOST_GATHER=$f,GLB_HOST_GATHER_THREADS=8,GLB_GATHER_BPS_PIPE=$b,GLB_HOST_GATHER_SCATTER_BLOCKS=$sb"
done; done; done
python tools/ab_env.py --config PA --alpha 0.22 --steps 40 --repeat 1 --variants "$V" > gpurun_out/hg_tune_PA.jsonl 2>&1
for mb in 0 148 64 32 16 8; do GLB_MISS_BLOCKS=$mb python tools/miss_probe.py --spans 1.0 --bins 21 --reps 3 > gpurun_out/missblocks_probe_$mb.jsonl 2>&1; done
V="zc:GLB_HOST_GATHER=0"
for mb in 148 64 32 16; do V="$V;zc_mb$mb:GLB_HOST_GATHER=0,GLB_MISS_BLOCKS=$mb;hg_mb$mb:GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8,GLB_MISS_BLOCKS=$mb"; done
python tools/ab_env.py --config PA --alpha 0.22 --steps 40 --repeat 1 --variants "$V" > gpurun_out/missblocks_PA.jsonl 2>&1
python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "extract" > gpurun_out/pytest_extract2.log 2>&1; tail -2 gpurun_out/pytest_extract2.log
