mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
nvidia-smi --query-gpu=utilization.gpu,memory.used,clocks.sm --format=csv
free -g | head -2
timeout 900 python bench.py --no-cpu --no-johnson --no-packed16 --steps 3 > gpurun_out/bench_e2e.json 2> gpurun_out/bench_e2e.err; tail -3 gpurun_out/bench_e2e.err; python -c "
import json; d=json.loads(open('gpurun_out/bench_e2e.json').read().strip().splitlines()[-1]); e=d['e2e']
print('i32', d['value'], 'e2e', e['value'], e['ms_per_step'], e['ms_parts_each_step'], e['serial']['ms_parts_each_step'])"
