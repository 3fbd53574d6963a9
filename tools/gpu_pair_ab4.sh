#!/bin/bash
# old tree vs current, pair off / on: int32 n = 16384, 32768, 65536; fp32 n = 32768
mkdir -p gpurun_out
(cd build/oldsrc && python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1)
{
for n in 16384 32768 65536; do
  r=3; d=4; [ $n -gt 16384 ] && r=2; [ $n -gt 32768 ] && r=1 && d=16
  echo "== old n=$n"; (cd build/oldsrc && python tools/fw_ab.py --n $n --deg $d --dtype i32 --runs $r --modes dataflow)
  for pair in 0 1; do echo "== new pair=$pair n=$n"; APSP_DF_PAIR=$pair python tools/fw_ab.py --n $n --deg $d --dtype i32 --runs $r --modes dataflow; done
done
echo "== old f32 n=32768"; (cd build/oldsrc && python tools/fw_ab.py --n 32768 --deg 64 --dtype f32 --runs 2 --modes dataflow)
for pair in 0 1; do echo "== new pair=$pair f32 n=32768"; APSP_DF_PAIR=$pair python tools/fw_ab.py --n 32768 --deg 64 --dtype f32 --runs 2 --modes dataflow; done
} > gpurun_out/pair_ab4.txt 2>&1
python3 - <<'PY'
import json
for l in open("gpurun_out/pair_ab4.txt"):
    if l.startswith("=="): print(l.strip(), end=" ")
    elif l.startswith("{"):
        d = json.loads(l)["dataflow"]; print("%.4f s  frac %.4f" % (d["device_s"], d["device_relax_per_s"] / 18.519e12))
PY
