set -x
python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "cold or extract_sample_bytes or generic_ids" > gpurun_out/pytest_cold.log 2>&1; tail -2 gpurun_out/pytest_cold.log
python tools/ab_env.py --config PA --alpha 0.22 --steps 30 --repeat 2 --variants "base:GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8;cold:GLB_COLD_STORE=1,GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8;cold_f150:GLB_COLD_STORE=1,GLB_HOST_GATHER=150,GLB_HOST_GATHER_THREADS=8;cold_f350:GLB_COLD_STORE=1,GLB_HOST_GATHER=350,GLB_HOST_GATHER_THREADS=8;cold_zc:GLB_COLD_STORE=1,GLB_HOST_GATHER=0" > gpurun_out/cold_PA.jsonl 2>&1
python tools/ab_env.py --config UK --alpha 0.18 --steps 20 --repeat 2 --variants "base:;cold:GLB_COLD_STORE=1" > gpurun_out/cold_UK.jsonl 2>&1
