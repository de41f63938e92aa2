set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python tools/sanitize.py > gpurun_out/sanitize_plain_r02m.log 2>&1; tail -1 gpurun_out/sanitize_plain_r02m.log
for T in memcheck racecheck synccheck; do
  echo "== $T"
  timeout 1500 compute-sanitizer --tool $T --print-limit 20 python tools/sanitize.py 2>&1 | tail -6
done > gpurun_out/sanitizer_r02m.txt 2>&1
cat gpurun_out/sanitizer_r02m.txt
