# packed16 dataflow kernel: tests, bench, A/B vs per-phase, 3-CTA variant.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_packed16.py -q -x > gpurun_out/pytest_p16.log 2>&1; tail -3 gpurun_out/pytest_p16.log
timeout 600 python tools/fw_ab.py --n 16384 --deg 8 --dtype i32 --packed16 --runs 2 2>&1 | tail -1
timeout 600 python tools/fw_ab.py --n 65536 --deg 16 --dtype i32 --packed16 --runs 1 --modes dataflow 2>&1 | tail -1
timeout 900 python bench.py --no-cpu --no-johnson > gpurun_out/bench_df16.json 2> gpurun_out/bench_df16.err; python -c "
import json; d=json.loads(open('gpurun_out/bench_df16.json').read().strip().splitlines()[-1]); p=d['packed16']; print('i32', d['value'], d['roofline']['frac']); print('p16', p['value'], p['roofline']['frac'], p['roofline']['kernel'], p['e2e']['value'])"
APSP_NVCC_EXTRA="-DDF16_CTAS=3" python -c "
import importlib.util
spec=importlib.util.spec_from_file_location('b','paper_conf_ipps_xia0ar22_b200/_build.py'); b=importlib.util.module_from_spec(spec); spec.loader.exec_module(b); b.build_lib(force=True)" > /dev/null
timeout 300 python -m pytest tests/test_gpu_packed16.py -q -x -k "dataflow or config1" 2>&1 | tail -1
timeout 600 python tools/fw_ab.py --n 16384 --deg 8 --dtype i32 --packed16 --runs 2 --modes dataflow 2>&1 | tail -1
