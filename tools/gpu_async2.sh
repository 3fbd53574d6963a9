mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_async.py tests/test_gpu_packed16.py -q -x > gpurun_out/pytest_async.log 2>&1; tail -15 gpurun_out/pytest_async.log
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; tail -3 gpurun_out/bench_full.err; python -c "
import json; d=json.loads(open('gpurun_out/bench_full.json').read().strip().splitlines()[-1]); e=d['e2e']; p=d['packed16']
print('i32', d['value'], d['roofline']['frac'], 'e2e', e['value'], e['ms_per_step'], e['ms_parts_each_step'], e['serial']['value'], e['serial']['ms_parts_each_step'])
print('p16', p['value'], p['roofline']['frac'], 'e2e', p['e2e']['value'], p['e2e']['serial']['value'])
print('cpu', d['cpu_baseline'])"
