python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
summ() { python -c "import json,sys; d=json.load(open(sys.argv[1])); r=d['roofline']; print(sys.argv[2], '%.4e'%d['value'], '%.1f ms'%d['ms_per_step'], 'frac %.3f'%r['frac'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" $1 "$2"; }
timeout 200 python bench.py --no-packed16 --no-cpu --no-e2e > gpurun_out/b.json 2>/dev/null; summ gpurun_out/b.json "df groups=2"
APSP_NVCC_EXTRA=-DDF_GROUPS=1 python -c "
import importlib.util
spec=importlib.util.spec_from_file_location('b','paper_conf_ipps_xia0ar22_b200/_build.py'); b=importlib.util.module_from_spec(spec); spec.loader.exec_module(b); b.build_lib(force=True)" > /dev/null
timeout 200 python -m pytest tests/test_gpu_dataflow.py -x -q 2>&1 | tail -1
APSP_DF_PROFILE=1 python tools/profile_fw.py --runs 1
for st in 0 16000; do APSP_DF_STAGGER=$st timeout 200 python bench.py --no-packed16 --no-cpu --no-e2e > gpurun_out/b.json 2>/dev/null; summ gpurun_out/b.json "df groups=1 stagger=$st"; done
