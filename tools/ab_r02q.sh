set -x
python tools/ab_env.py --config PA --alpha 0.22 --steps 30 --repeat 3 --variants "base:GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8;xhigh:GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8,GLB_XSTREAM_HIGH=1;xhigh_pipe4:GLB_HOST_GATHER=250,GLB_HOST_GATHER_THREADS=8,GLB_XSTREAM_HIGH=1,GLB_GATHER_BPS_PIPE=4" > gpurun_out/prio_PA.jsonl 2>&1
python tools/ab_env.py --config PR --alpha 1.0 --steps 200 --repeat 2 --variants "base:;xhigh:GLB_XSTREAM_HIGH=1" > gpurun_out/prio_PR.jsonl 2>&1
