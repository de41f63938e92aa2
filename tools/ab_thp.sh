# host feature memory: pageable + cudaHostRegister (4 KB pages), THP (madvise 2 MB) + register, cudaHostAlloc
for C in "PA 0.22 512" "UK 0.18 1024"; do set -- $C
for A in register thp cuda; do
  timeout 900 python bench.py --config $1 --alpha $2 --steps 40 --warmup 3 --no-sweep --no-cpu-baseline --k-sweep "" --host-alloc $A | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); u=d['units']; print('$1 alloc=$A', round(d['value']/1e6,3), 'extract ms', round(d['roofline']['extract_ms_per_step'],3), 'misses', round(u['mean_misses']), 'GB/s', round(u['mean_misses']*$3/d['roofline']['extract_ms_per_step']/1e6,1), d['preprocess_s'])"
done; done
grep -i AnonHugePages /proc/meminfo; cat /sys/kernel/mm/transparent_hugepage/enabled
