# r02i2: an L2-sized relabel hash table (capacity 2^21-2^22 entries, ~2.5-3.5x the sample's
# unique vertices, 40-80 MB with the slots) with and without a persisting L2 window, against
# the dense table, on the big graphs at alpha = 1 (the sampler-heavy steps)
set -x
for C in TW UK PA; do
  python tools/ab_env.py --config $C --alpha 1.0 --steps 40 --repeat 2 --relabel dense \
      --variants "dense:;dense_pin0:GLB_L2_PIN=0" > gpurun_out/l2hash_dense_${C}.jsonl 2>&1
  python tools/ab_env.py --config $C --alpha 1.0 --steps 40 --repeat 2 --relabel hash \
      --variants "h22:GLB_HASH_LOG2=22,GLB_L2_PIN=0;h22pin:GLB_HASH_LOG2=22,GLB_L2_PIN=1;h21pin:GLB_HASH_LOG2=21,GLB_L2_PIN=1;hbound:" > gpurun_out/l2hash_hash_${C}.jsonl 2>&1
done
