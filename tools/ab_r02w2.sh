# r02w2: cold store on TW (1 KB rows) at the paper's R% -- does the <= 512-byte auto rule hold?
set -x
python tools/ab_env.py --config TW --alpha 0.25 --steps 20 --repeat 3 --variants "gid:GLB_COLD_STORE=0;cold:GLB_COLD_STORE=1" > gpurun_out/cold_TW_r02w2.jsonl 2>&1
