mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_async.py tests/test_gpu_packed16.py -q -x 2>&1 | tail -3
timeout 900 python bench.py --no-cpu --no-johnson > gpurun_out/bench.json 2> gpurun_out/bench.err; python -c "
import json; d=json.loads(open('gpurun_out/bench.json').read().strip().splitlines()[-1]); p=d['packed16']
print('i32', d['value'], d['roofline']['frac'], 'e2e', d['e2e']['value']); print('p16', p['value'], p['roofline']['frac'], 'e2e', p['e2e']['value'], p['e2e']['ms_per_step'])"
