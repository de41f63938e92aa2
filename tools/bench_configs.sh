# bench lines for the other BASELINE configs (paper R% alpha and alpha=1) + weighted shapes
for C in "TW 0.25" "TW 1.0" "PA 0.22" "PA 1.0" "UK 0.18" "UK 1.0" "PRW 1.0" "TWW 1.0"; do
  set -- $C
  echo "== $1 alpha=$2"
  timeout 900 python bench.py --config $1 --alpha $2 --steps 60 --warmup 3 --sweep-steps 4 --cpu-seconds 10 2>&1 | tail -1
done
