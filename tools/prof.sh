set -x
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_r01.csv python bench.py --steps 10 --warmup 3 --no-sweep --no-cpu-baseline > gpurun_out/b_ncu.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_gather -s 30 -c 2 -o gpurun_out/prof_gather python bench.py --steps 10 --warmup 3 --no-sweep --no-cpu-baseline > gpurun_out/p1.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_compact -s 60 -c 2 -o gpurun_out/prof_compact python bench.py --steps 10 --warmup 3 --no-sweep --no-cpu-baseline > gpurun_out/p2.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_khop -s 30 -c 2 -o gpurun_out/prof_khop python bench.py --steps 10 --warmup 3 --no-sweep --no-cpu-baseline > gpurun_out/p3.log 2>&1
ls -la gpurun_out
