# r02d: why the launch list of the default bench died (rc 9) under ncu with the host-assisted
# part on: host memory headroom, then the launch list again with the kernel log checked.
set -x
TAG=${1:-r02d}
free -g; nproc
B0="python bench.py --steps 4 --warmup 3 --runs 1 --no-sweep --no-cpu-baseline --no-pr-alpha1"
/usr/bin/time -v $B0 > gpurun_out/plain_$TAG.json 2> gpurun_out/plain_$TAG.err; grep -E "Maximum resident|Exit status" gpurun_out/plain_$TAG.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv --log-file gpurun_out/launches_$TAG.csv \
    $B0 > gpurun_out/launches_$TAG.log 2>&1; echo "rc=$?"; tail -3 gpurun_out/launches_$TAG.log
dmesg 2>/dev/null | tail -5
ncu --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv --log-file gpurun_out/launches_nocold_$TAG.csv \
    $B0 --cold-store off > gpurun_out/launches_nocold_$TAG.log 2>&1; echo "rc=$?"; tail -3 gpurun_out/launches_nocold_$TAG.log
