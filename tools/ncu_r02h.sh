# r02h: ncu counters of k_gather (3 launches, depth 1, serialised) for the configs whose bench
# lines had no `traffic` yet: every big graph at alpha = 1 (HBM-bound) and TWW at the paper's R%
set -x
TAG=${1:-r02h}
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,pcie__read_bytes.sum,pcie__write_bytes.sum,syslts__t_sectors_aperture_sysmem_op_read.sum,syslts__t_requests_aperture_sysmem_op_read.sum
for C in "PA 1.0" "TW 1.0" "UK 1.0" "PRW 1.0" "TWW 1.0" "TWW 0.25"; do
  set -- $C
  ncu --metrics $M --clock-control none --cache-control none -k regex:k_gather -s 4 -c 3 --csv \
      --log-file gpurun_out/hostlink_${1}_${2}_$TAG.csv \
      python bench.py --config $1 --alpha $2 --steps 4 --warmup 3 --runs 1 --no-sweep --no-cpu-baseline --no-pr-alpha1 --pipeline 1 \
      > gpurun_out/ncu_${1}_${2}_$TAG.log 2>&1; echo "$C rc=$?"
done
