# async serving API: tests, bench (pipelined e2e), packed16 3-CTA variant.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_async.py -q -x > gpurun_out/pytest_async.log 2>&1; tail -15 gpurun_out/pytest_async.log
timeout 900 python bench.py --no-cpu --no-johnson > gpurun_out/bench_async.json 2> gpurun_out/bench_async.err; tail -3 gpurun_out/bench_async.err; python -c "
import json; d=json.loads(open('gpurun_out/bench_async.json').read().strip().splitlines()[-1]); p=d['packed16']
print('i32', d['value'], d['roofline']['frac'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'], d['e2e']['serial'])
print('p16', p['value'], p['roofline']['frac'], 'e2e', p['e2e']['value'], p['e2e']['serial']['value'])"
APSP_NVCC_EXTRA="-DDF16_CTAS=3" python -c "
import importlib.util
spec=importlib.util.spec_from_file_location('b','paper_conf_ipps_xia0ar22_b200/_build.py'); b=importlib.util.module_from_spec(spec); spec.loader.exec_module(b); b.build_lib(force=True)" > /dev/null
echo "== DF16_CTAS=3"
timeout 300 python -m pytest tests/test_gpu_packed16.py -q -x -k "dataflow or config1" 2>&1 | tail -1
timeout 600 python tools/fw_ab.py --n 16384 --deg 8 --dtype i32 --packed16 --runs 2 --modes dataflow 2>&1 | tail -1
