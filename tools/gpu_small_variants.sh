#!/bin/bash
# small-n kernel tuning: queue variant (decode_fuse default, decode without fusion) x CTAs per SM
# x n, against the 128-tile dataflow kernel
mkdir -p gpurun_out
for n in 1024 1536 2048 3072 4096; do
  echo "== n=$n dataflow128"; python tools/fw_ab.py --n $n --deg 8 --dtype i32 --runs 20 --modes dataflow
  for v in decode_fuse decode; do for c in 1 2 3; do
    echo "== n=$n queue=$v ctas=$c"
    APSP_SMALL_QUEUE=$v APSP_SMALL_CTAS=$c python tools/fw_ab.py --n $n --deg 8 --dtype i32 --runs 20 --modes small
  done; done
done > gpurun_out/small_variants.txt 2>&1
python3 - <<'PY'
import json
for l in open("gpurun_out/small_variants.txt"):
    if l.startswith("=="): print(l.strip(), end=" ")
    elif l.startswith("{"):
        d = json.loads(l); k = "small" if "small" in d else "dataflow"; print(round(d[k]["device_s"] * 1e3, 4), "ms")
PY
