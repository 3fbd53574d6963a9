# A/B: own-element C loads (no epilogue barrier) and the next-chunk prefetch for int32
mkdir -p gpurun_out
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], '%.4e'%d['value'], '%.2f ms'%d['ms_per_step'], 'frac %.4f'%r['frac'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" $1 "$2"; }
rebuild() { APSP_NVCC_EXTRA="$1" python -c "
import importlib.util
spec=importlib.util.spec_from_file_location('b','paper_conf_ipps_xia0ar22_b200/_build.py'); b=importlib.util.module_from_spec(spec); spec.loader.exec_module(b); b.build_lib(force=True)" > /dev/null; }
for rep in 1 2; do
for v in "base:" "ownc:-DDF_OWNC" "ownc_xall:-DDF_OWNC -DDF_XPREF_ALL"; do
  name="${v%%:*}"; flags="${v#*:}"
  rebuild "$flags"
  if [ $rep = 1 ] && [ $name != base ]; then timeout 600 python -m pytest tests/test_gpu_dataflow.py tests/test_gpu_parity.py -q -x 2>&1 | tail -1; fi
  timeout 300 python bench.py --no-packed16 --no-cpu --no-e2e --no-johnson --steps 5 > gpurun_out/b.json 2>/dev/null; summ gpurun_out/b.json "$name"
  timeout 600 python tools/fw_ab.py --n 32768 --deg 64 --dtype f32 --runs 1 --modes dataflow 2>&1 | tail -1 | cut -c60-130
done
done
rebuild ""
