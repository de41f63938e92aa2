# hot-first renumbering experiment: original vs renumbered graph, pipelined step
for C in TW UK; do
  timeout 900 python tools/hotfirst.py $C orig
  timeout 900 python tools/hotfirst.py $C hot
done
