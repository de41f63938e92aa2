# L2 prefetch-size hints on the gather's row loads (GLB_GATHER_LD=3: .L2::64B, 4: .L2::256B) and on the
# sampler's random CSR reads (GLB_SAMPLE_LD=1: .L2::64B), A/B builds, pipeline depth 2
set -x
for C in "PR 1.0 200" "UK 1.0 60" "TW 1.0 60" "PA 0.22 30"; do
  set -- $C
  for L in default WT_ld3 WT_ld4 WT_sld1 WT_ld3sld1; do
    if [ $L = default ]; then unset GLB_LIBRARY; else export GLB_LIBRARY=build/ab/libglb_$L.so; fi
    HG=""; [ $1 = PA ] && HG="--host-gather 0.25"
    python tools/ab_env.py --config $1 --alpha $2 --steps $3 --repeat 2 $HG --variants "$L:" >> gpurun_out/ldhint_$1.jsonl 2>&1
  done
  unset GLB_LIBRARY
done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for L in default WT_ld3 WT_ld4; do
  if [ $L = default ]; then unset GLB_LIBRARY; else export GLB_LIBRARY=build/ab/libglb_$L.so; fi
  ncu --metrics $M --clock-control none --cache-control none -k "regex:k_gather|k_khop|k_compact" -s 101 -c 15 --csv \
      --log-file gpurun_out/ldhint_ncu_PR_$L.csv python bench.py --config PR --steps 4 --warmup 3 --runs 1 --no-sweep --no-cpu-baseline --pipeline 1 > /dev/null 2>&1
done
unset GLB_LIBRARY
