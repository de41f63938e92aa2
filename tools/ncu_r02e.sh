# r02e: the launch list of the default bench command (cold store on) and the host-link counters of
# its extract kernels with the host-assisted part on.  Kernel replay makes ncu back up the
# registered host memory the kernels can reach (57 GB matrix + 44 GB cold store) and the box
# (196 GB) runs out (rc 9, r02d); application replay re-runs the program per pass instead.
set -x
TAG=${1:-r02e}
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,pcie__read_bytes.sum,pcie__write_bytes.sum,syslts__t_sectors_aperture_sysmem_op_read.sum,syslts__t_requests_aperture_sysmem_op_read.sum
B0="python bench.py --steps 4 --warmup 3 --runs 1 --no-sweep --no-cpu-baseline --no-pr-alpha1"
ncu --replay-mode application --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv \
    --log-file gpurun_out/launches_$TAG.csv $B0 > gpurun_out/launches_$TAG.log 2>&1; echo "rc=$?"
ncu --replay-mode application --metrics $M --clock-control none --cache-control none -k "regex:k_gather|k_hg_scatter" -s 8 -c 10 --csv \
    --log-file gpurun_out/hostlink_PA_cold_hg_$TAG.csv $B0 --pipeline 1 > gpurun_out/ncu_hostlink_PA_cold_hg_$TAG.log 2>&1; echo "rc=$?"
