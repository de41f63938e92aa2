# r02t: 64-byte L2 fill on the sampler's random indptr loads (default build) vs plain loads
# (GLB_INDPTR_LD=0 build), alpha = 1 on every shape (the sampler-heavy steps), alternating builds
set -x
for C in "PR 1.0 200" "TW 1.0 60" "UK 1.0 60" "PA 1.0 60"; do
  set -- $C
  for L in default WT_ip0 default WT_ip0; do
    if [ $L = default ]; then unset GLB_LIBRARY; else export GLB_LIBRARY=build/ab/libglb_$L.so; fi
    python tools/ab_env.py --config $1 --alpha $2 --steps $3 --repeat 2 --variants "$L:" >> gpurun_out/indptr_ld_$1.jsonl 2>&1
  done
  unset GLB_LIBRARY
done
