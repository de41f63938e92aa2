# r02c: ncu evidence for the headline with the cold store (bench defaults: PA, alpha 0.22,
# cold store on, host-assisted share 0.15).  (1) launch list of the bench command;
# (2) host-link counters of the extract kernels in the bench's configuration at depth 1;
# (3) the same zero-copy only (--host-gather 0) with the cold store; (4) --set full of k_gather.
set -x
TAG=${1:-r02c}
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,pcie__read_bytes.sum,pcie__write_bytes.sum,syslts__t_sectors_aperture_sysmem_op_read.sum,syslts__t_requests_aperture_sysmem_op_read.sum
B0="python bench.py --steps 4 --warmup 3 --runs 1 --no-sweep --no-cpu-baseline --no-pr-alpha1"
ncu --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv --log-file gpurun_out/launches_$TAG.csv \
    $B0 > gpurun_out/launches_$TAG.log 2>&1
ncu --metrics $M --clock-control none --cache-control none -k "regex:k_gather|k_hg_scatter" -s 8 -c 10 --csv \
    --log-file gpurun_out/hostlink_PA_cold_hg_$TAG.csv $B0 --pipeline 1 > gpurun_out/ncu_hostlink_PA_cold_hg_$TAG.log 2>&1
ncu --metrics $M --clock-control none --cache-control none -k regex:k_gather -s 4 -c 3 --csv \
    --log-file gpurun_out/hostlink_PA_cold_$TAG.csv $B0 --pipeline 1 --host-gather 0 > gpurun_out/ncu_hostlink_PA_cold_$TAG.log 2>&1
ncu --set full --clock-control none --cache-control none --import-source on -k regex:k_gather -s 4 -c 1 \
    -o gpurun_out/prof_k_gather_PA_cold_$TAG $B0 --pipeline 1 --host-gather 0 > gpurun_out/ncu_full_PA_cold_$TAG.log 2>&1
ls -la gpurun_out | tail
