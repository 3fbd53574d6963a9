# dataflow kernel sweeps on cfg2: queue delay (runtime) and phase-3 band width (compile time)
mkdir -p gpurun_out
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], '%.4e'%d['value'], '%.2f ms'%d['ms_per_step'], 'frac %.4f'%r['frac'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" $1 "$2"; }
rebuild() { APSP_NVCC_EXTRA="$1" python -c "
import importlib.util
spec=importlib.util.spec_from_file_location('b','paper_conf_ipps_xia0ar22_b200/_build.py'); b=importlib.util.module_from_spec(spec); spec.loader.exec_module(b); b.build_lib(force=True)" > /dev/null; }
rebuild ""
for d in 0 148 592 2368 4736; do
  timeout 300 python bench.py --no-packed16 --no-cpu --no-e2e --no-johnson --df-delay $d --steps 5 > gpurun_out/b.json 2>/dev/null; summ gpurun_out/b.json "delay=$d"
done
for band in 16 32 128; do
  rebuild "-DDF_BAND=$band"
  timeout 300 python bench.py --no-packed16 --no-cpu --no-e2e --no-johnson --steps 5 > gpurun_out/b.json 2>/dev/null; summ gpurun_out/b.json "band=$band"
done
rebuild ""
timeout 300 python bench.py --no-packed16 --no-cpu --no-e2e --no-johnson --steps 5 > gpurun_out/b.json 2>/dev/null; summ gpurun_out/b.json "base again"
