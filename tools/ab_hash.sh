for H in "" 21; do
  GLB_HASH_LOG2=$H timeout 300 python bench.py --config UK --relabel hash --alpha 1.0 --steps 60 --no-sweep --no-cpu-baseline | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('UK hash log2=$H', round(d['value']/1e6,2), round(d['ms_per_step']*1e3,1), 'us/step extract', round(d['roofline']['extract_ms_per_step']*1e3,1))"
done
GLB_HASH_LOG2=21 timeout 600 ncu --metrics gpu__time_duration.sum,lts__t_sector_hit_rate.pct,dram__bytes_read.sum --clock-control none --cache-control none -c 120 --csv --log-file gpurun_out/launches_uk_h21.csv python bench.py --config UK --alpha 1.0 --steps 4 --warmup 2 --no-sweep --no-cpu-baseline --relabel hash > /dev/null 2>&1
echo done
