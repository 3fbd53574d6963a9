# A/B of the dataflow kernel vs the launch-per-phase schedule on the bench workload (gpurun).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
timeout 300 python -m pytest tests/test_gpu_dataflow.py -x -q > gpurun_out/df_tests.log 2>&1; echo rc=$? >> gpurun_out/df_tests.log; tail -2 gpurun_out/df_tests.log
APSP_NVCC_EXTRA=-DDF_PROF=1 python -c "
import importlib.util
spec=importlib.util.spec_from_file_location('b','paper_conf_ipps_xia0ar22_b200/_build.py'); b=importlib.util.module_from_spec(spec); spec.loader.exec_module(b); b.build_lib(force=True)" > /dev/null
APSP_DF_PROFILE=1 python tools/profile_fw.py --runs 2
python -c "
import importlib.util
spec=importlib.util.spec_from_file_location('b','paper_conf_ipps_xia0ar22_b200/_build.py'); b=importlib.util.module_from_spec(spec); spec.loader.exec_module(b); b.build_lib(force=True)" > /dev/null
summ() { python -c "import json,sys; d=json.load(open(sys.argv[1])); r=d['roofline']; print(sys.argv[2], '%.4e'%d['value'], '%.1f ms'%d['ms_per_step'], 'frac %.3f'%r['frac'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" $1 "$2"; }
for st in ${STAGGERS:-0}; do
  APSP_DF_STAGGER=$st timeout 200 python bench.py --no-packed16 --no-cpu --no-e2e > gpurun_out/b.json 2>>gpurun_out/sweep.err
  summ gpurun_out/b.json "dataflow stagger=$st"
done
timeout 200 python bench.py --no-packed16 --no-cpu --no-e2e --legacy > gpurun_out/b.json 2>>gpurun_out/sweep.err; summ gpurun_out/b.json legacy
