#!/bin/bash
# two-round (pair) queue vs one-round queue, 128-tile dataflow kernel: int32 n=16384 / 65536, fp32 n=32768
mkdir -p gpurun_out
{
for pair in 0 1 0 1; do echo "== pair=$pair n=16384 i32"; APSP_DF_PAIR=$pair python tools/fw_ab.py --n 16384 --deg 4 --dtype i32 --runs 3 --modes dataflow; done
for pair in 0 1; do echo "== pair=$pair n=65536 i32"; APSP_DF_PAIR=$pair python tools/fw_ab.py --n 65536 --deg 16 --dtype i32 --runs 1 --modes dataflow; done
for pair in 0 1; do echo "== pair=$pair n=32768 f32"; APSP_DF_PAIR=$pair python tools/fw_ab.py --n 32768 --deg 64 --dtype f32 --runs 2 --modes dataflow; done
} > gpurun_out/pair_ab.txt 2>&1
python3 - <<'PY'
import json
for l in open("gpurun_out/pair_ab.txt"):
    if l.startswith("=="): print(l.strip(), end=" ")
    elif l.startswith("{"):
        d = json.loads(l)["dataflow"]; print("%.4f s  device %.4e relax/s  frac %.4f" % (d["device_s"], d["device_relax_per_s"], d["device_relax_per_s"] / 18.519e12))
PY
