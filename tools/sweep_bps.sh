# gather blocks-per-SM x pipeline depth sweep on the bench config
for P in 1 2; do for B in 2 3 4; do
  echo "pipeline=$P bps=$B"; GLB_GATHER_BPS=$B python bench.py --steps 400 --warmup 5 --no-sweep --no-cpu-baseline --pipeline $P | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e6,2),'Mseeds/s', round(d['ms_per_step']*1e3,1),'us/step', 'extract', round(d['roofline']['extract_ms_per_step']*1e3,1),'us', round(d['roofline']['frac'],3), d['clocks'])"
done; done
