python - <<'PY'
import torch
p=torch.cuda.get_device_properties(0)
print("persisting L2 max", torch.cuda.get_device_properties(0).L2_cache_size)
PY
for PIN in 1 0; do for C in "PR dense" "UK dense" "UK hash" "PA hash" "PA dense"; do set -- $C
  GLB_L2_PIN=$PIN python bench.py --config $1 --relabel $2 --alpha 1.0 --steps 60 --no-sweep --no-cpu-baseline | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('pin=$PIN', '$1', '$2', round(d['value']/1e6,2), round(d['ms_per_step']*1e3,1), 'us/step extract', round(d['roofline']['extract_ms_per_step']*1e3,1))"
done; done
