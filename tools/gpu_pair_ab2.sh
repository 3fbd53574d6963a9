#!/bin/bash
# A/B of the dataflow kernel: the pre-pair source tree (build/oldsrc, built here) vs the current
# tree with the pair queue on / off, int32 n = 16384 / 32768 / 65536, fp32 n = 32768
mkdir -p gpurun_out
(cd build/oldsrc && python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1)
{
for n in 16384 32768; do
  r=3; [ $n -gt 16384 ] && r=2
  echo "== old n=$n"; (cd build/oldsrc && python tools/fw_ab.py --n $n --deg 4 --dtype i32 --runs $r --modes dataflow)
  for pair in 0 1; do echo "== new pair=$pair n=$n"; APSP_DF_PAIR=$pair python tools/fw_ab.py --n $n --deg 4 --dtype i32 --runs $r --modes dataflow; done
done
echo "== old n=65536"; (cd build/oldsrc && python tools/fw_ab.py --n 65536 --deg 16 --dtype i32 --runs 1 --modes dataflow)
for pair in 0 1; do echo "== new pair=$pair n=65536"; APSP_DF_PAIR=$pair python tools/fw_ab.py --n 65536 --deg 16 --dtype i32 --runs 1 --modes dataflow; done
echo "== old n=32768 f32"; (cd build/oldsrc && python tools/fw_ab.py --n 32768 --deg 64 --dtype f32 --runs 2 --modes dataflow)
for pair in 0 1; do echo "== new pair=$pair n=32768 f32"; APSP_DF_PAIR=$pair python tools/fw_ab.py --n 32768 --deg 64 --dtype f32 --runs 2 --modes dataflow; done
} > gpurun_out/pair_ab2.txt 2>&1
python3 - <<'PY'
import json
for l in open("gpurun_out/pair_ab2.txt"):
    if l.startswith("=="): print(l.strip(), end=" ")
    elif l.startswith("{"):
        d = json.loads(l)["dataflow"]; print("%.4f s  device %.4e relax/s  frac %.4f" % (d["device_s"], d["device_relax_per_s"], d["device_relax_per_s"] / 18.519e12))
PY
