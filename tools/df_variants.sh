# Build and time compile-time variants of the dataflow kernel (gpurun experiments).
# usage: VARIANTS="base:| noacq:-DDF_NOACQ ..." bash tools/df_variants.sh
mkdir -p gpurun_out
summ() { python -c "import json,sys; d=json.load(open(sys.argv[1])); r=d['roofline']; print(sys.argv[2], '%.4e'%d['value'], '%.1f ms'%d['ms_per_step'], 'frac %.3f'%r['frac'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" $1 "$2"; }
rebuild() { APSP_NVCC_EXTRA="$1" python -c "
import importlib.util
spec=importlib.util.spec_from_file_location('b','paper_conf_ipps_xia0ar22_b200/_build.py'); b=importlib.util.module_from_spec(spec); spec.loader.exec_module(b); b.build_lib(force=True)" > /dev/null; }
IFS='|' read -ra VS <<< "${VARIANTS:-base:}"
for v in "${VS[@]}"; do
  name="${v%%:*}"; flags="${v#*:}"
  rebuild "$flags"
  timeout 200 python -m pytest tests/test_gpu_dataflow.py -x -q 2>&1 | tail -1
  timeout 200 python bench.py --no-packed16 --no-cpu --no-e2e ${BENCH_ARGS} > gpurun_out/b.json 2>>gpurun_out/var.err; summ gpurun_out/b.json "$name [$flags]"
done
rebuild ""
