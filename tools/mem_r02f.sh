# r02f: host memory headroom of the default bench command (MemAvailable sampled every second)
set -x
TAG=${1:-r02f}
( while true; do echo "$(date +%s) $(grep MemAvailable /proc/meminfo | awk '{print $2}')"; sleep 1; done ) > gpurun_out/memavail_$TAG.txt &
MP=$!
python bench.py --steps 8 --warmup 3 --runs 1 --no-sweep --no-pr-alpha1 > gpurun_out/mem_bench_$TAG.json 2> gpurun_out/mem_bench_$TAG.err
echo "rc=$?"
kill $MP
sort -k2 -n gpurun_out/memavail_$TAG.txt | head -3
