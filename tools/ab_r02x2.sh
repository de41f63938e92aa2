# r02x2: PA's random walks (k_rwalk) with plain index loads (GLB_SAMPLE_LD=0 build) vs the 64-byte fill
# (default), alpha = 1, builds alternated
set -x
for L in default WT_sld0 default WT_sld0; do
  if [ $L = default ]; then unset GLB_LIBRARY; else export GLB_LIBRARY=build/ab/libglb_$L.so; fi
  python tools/ab_env.py --config PA --alpha 1.0 --steps 60 --repeat 2 --variants "$L:" >> gpurun_out/sld_PA.jsonl 2>&1
done
