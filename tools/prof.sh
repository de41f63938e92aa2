# Per-kernel launch list + full ncu captures of the hot kernels (bench config, 1 GPU).
# usage: bash tools/prof.sh <tag>
set -x
TAG=${1:-r01}
B="python bench.py --steps 10 --warmup 3 --no-sweep --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -c 300 --csv --log-file gpurun_out/launches_$TAG.csv $B > gpurun_out/b_ncu_$TAG.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_gather -s 20 -c 1 -o gpurun_out/prof_gather_$TAG $B > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_compact -s 40 -c 2 -o gpurun_out/prof_compact_$TAG $B > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_khop -s 20 -c 2 -o gpurun_out/prof_khop_$TAG $B > /dev/null 2>&1
ls -la gpurun_out
