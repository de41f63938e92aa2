# A/B of the host-assisted miss gather (glb_set_host_gather) on the miss-heavy configs
set -x
python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "extract or host_gather or pipeline" > gpurun_out/pytest_hg.log 2>&1; tail -3 gpurun_out/pytest_hg.log
GLB_HOST_GATHER_DMA=1 python tools/miss_ab.py --config PA --alpha 0.22 --bins 21 --hg 0,150,250,350,450 --hg-threads 14 > gpurun_out/hg_PA_dma.jsonl 2>&1
GLB_HOST_GATHER_DMA=0 python tools/miss_ab.py --config PA --alpha 0.22 --bins 21 --hg 150,250 --hg-threads 14 > gpurun_out/hg_PA_zc.jsonl 2>&1
GLB_HOST_GATHER_DMA=1 python tools/miss_ab.py --config UK --alpha 0.18 --bins 21 --hg 0,150,300 --hg-threads 14 > gpurun_out/hg_UK_dma.jsonl 2>&1
