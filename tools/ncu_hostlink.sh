# ncu host-link evidence for the extract on the miss-heavy configs at the paper's R%:
# per-launch DRAM bytes, PCIe read bytes and sysmem L2 sectors of k_gather (zero-copy
# misses only: --host-gather 0), the same with the host-assisted part on (PA: k_gather +
# k_hg_scatter), and one --set full capture of PA's gather.
# usage: bash tools/ncu_hostlink.sh <tag> [configs]
set -x
TAG=${1:-r02}
CONFIGS=${2:-"PA TW UK"}
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,pcie__read_bytes.sum,pcie__write_bytes.sum,syslts__t_sectors_aperture_sysmem_op_read.sum,syslts__t_requests_aperture_sysmem_op_read.sum
for C in $CONFIGS; do
  B="python bench.py --config $C --steps 4 --warmup 3 --runs 1 --no-sweep --no-cpu-baseline --no-pr-alpha1 --pipeline 1 --host-gather 0"
  ncu --metrics $M --clock-control none --cache-control none -k regex:k_gather -s 4 -c 3 --csv \
      --log-file gpurun_out/hostlink_${C}_$TAG.csv $B > gpurun_out/ncu_hostlink_${C}_$TAG.log 2>&1
done
B="python bench.py --config PA --steps 4 --warmup 3 --runs 1 --no-sweep --no-cpu-baseline --no-pr-alpha1 --pipeline 2"
ncu --metrics $M --clock-control none --cache-control none -k "regex:k_gather|k_hg_scatter" -s 8 -c 10 --csv \
    --log-file gpurun_out/hostlink_PA_hg_$TAG.csv $B > gpurun_out/ncu_hostlink_PA_hg_$TAG.log 2>&1
B="python bench.py --config PA --steps 4 --warmup 3 --runs 1 --no-sweep --no-cpu-baseline --no-pr-alpha1 --pipeline 1 --host-gather 0"
ncu --set full --clock-control none --cache-control none --import-source on -k regex:k_gather -s 4 -c 1 \
    -o gpurun_out/prof_k_gather_PA_$TAG $B > gpurun_out/ncu_full_PA_$TAG.log 2>&1
ls -la gpurun_out | tail
