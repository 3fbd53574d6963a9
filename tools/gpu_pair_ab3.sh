#!/bin/bash
# does the presence of the pair code slow the one-round kernel? old tree vs current built with
# -DDF_NO_PAIR_CODE vs current (pair off / on), int32 n = 16384 and 65536
mkdir -p gpurun_out
(cd build/oldsrc && python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1)
rm -rf /tmp/nopair && cp -r . /tmp/nopair && (cd /tmp/nopair && rm -f build/obj/apsp_fw_dataflow.cu.o && APSP_NVCC_EXTRA=-DDF_NO_PAIR_CODE python -c "
import importlib.util; spec = importlib.util.spec_from_file_location('b', 'paper_conf_ipps_xia0ar22_b200/_build.py'); b = importlib.util.module_from_spec(spec); spec.loader.exec_module(b); b.build_lib(force=True)" > /dev/null 2>&1)
{
for n in 16384 65536; do
  r=3; d=4; [ $n -gt 16384 ] && r=1 && d=16
  echo "== old n=$n"; (cd build/oldsrc && python tools/fw_ab.py --n $n --deg $d --dtype i32 --runs $r --modes dataflow)
  echo "== nopair n=$n"; (cd /tmp/nopair && python tools/fw_ab.py --n $n --deg $d --dtype i32 --runs $r --modes dataflow)
  for pair in 0 1; do echo "== new pair=$pair n=$n"; APSP_DF_PAIR=$pair python tools/fw_ab.py --n $n --deg $d --dtype i32 --runs $r --modes dataflow; done
done
} > gpurun_out/pair_ab3.txt 2>&1
python3 - <<'PY'
import json
for l in open("gpurun_out/pair_ab3.txt"):
    if l.startswith("=="): print(l.strip(), end=" ")
    elif l.startswith("{"):
        d = json.loads(l)["dataflow"]; print("%.4f s  device %.4e relax/s  frac %.4f" % (d["device_s"], d["device_relax_per_s"], d["device_relax_per_s"] / 18.519e12))
PY
