# gather register budget / loads in flight per thread (A/B builds: GLB_GATHER_VEC, GLB_GATHER_MINB)
set -x
for C in "PR 1.0 200" "UK 1.0 60" "PA 0.22 30"; do
  set -- $C
  for L in default WT_v16m2 WT_v12m2 WT_v8m2 WT_v4m4; do
    if [ $L = default ]; then unset GLB_LIBRARY; else export GLB_LIBRARY=build/ab/libglb_$L.so; fi
    HG=""; [ $1 = PA ] && HG="--host-gather 0.25"
    python tools/ab_env.py --config $1 --alpha $2 --steps $3 --repeat 2 $HG --variants "$L:" >> gpurun_out/gather_regs_$1.jsonl 2>&1
  done
  unset GLB_LIBRARY
done
