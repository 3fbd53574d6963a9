#!/bin/bash
# small-n kernel tuning: queue delay (G3R(k-1) tasks before round k's panels) x n
mkdir -p gpurun_out
for n in 1024 2048; do for d in 1 16 32 64 128 256; do
  echo "== n=$n delay=$d"
  python tools/fw_ab.py --n $n --deg 8 --dtype i32 --runs 30 --modes small --delay $d
done; done > gpurun_out/small_variants.txt 2>&1
python3 - <<'PY'
import json
for l in open("gpurun_out/small_variants.txt"):
    if l.startswith("=="): print(l.strip(), end=" ")
    elif l.startswith("{"):
        d = json.loads(l); k = "small" if "small" in d else "dataflow"; print(round(d[k]["device_s"] * 1e3, 4), "ms")
PY
