set -x
python bench.py --steps 20 --warmup 5 --no-sweep --no-cpu-baseline --no-pr-alpha1 > gpurun_out/m_a.json 2>/dev/null
python bench.py --steps 20 --warmup 5 --no-sweep --no-cpu-baseline --no-pr-alpha1 --time-every 1 > gpurun_out/m_b.json 2>/dev/null
python bench.py --steps 60 --warmup 5 --runs 1 --no-sweep --no-cpu-baseline --no-pr-alpha1 > gpurun_out/m_c.json 2>/dev/null
python bench.py --steps 20 --warmup 5 --no-sweep --no-cpu-baseline --no-pr-alpha1 --time-every 1 > gpurun_out/m_d.json 2>/dev/null
