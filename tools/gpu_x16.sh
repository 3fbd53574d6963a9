# A/B: packed16 dataflow kernel with the next-chunk prefetch (-DDF16_XPREF)
mkdir -p gpurun_out
rebuild() { APSP_NVCC_EXTRA="$1" python -c "
import importlib.util
spec=importlib.util.spec_from_file_location('b','paper_conf_ipps_xia0ar22_b200/_build.py'); b=importlib.util.module_from_spec(spec); spec.loader.exec_module(b); b.build_lib(force=True)" > /dev/null; }
for rep in 1 2; do
for v in "base:" "x16:-DDF16_XPREF"; do
  name="${v%%:*}"; flags="${v#*:}"
  rebuild "$flags"
  if [ $rep = 1 ] && [ $name = x16 ]; then timeout 600 python -m pytest tests/test_gpu_packed16.py -q -x 2>&1 | tail -1; fi
  echo "$name"; timeout 600 python tools/fw_ab.py --n 16384 --deg 8 --dtype i32 --packed16 --runs 2 --modes dataflow 2>&1 | tail -1 | cut -c60-150
done
done
rebuild ""
