mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], '%.4e'%d['value'], '%.2f ms'%d['ms_per_step'], 'frac %.4f'%r['frac'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" $1 "$2"; }
timeout 600 python -m pytest tests/test_gpu_dataflow.py tests/test_gpu_sharded.py tests/test_gpu_parity.py tests/test_gpu_async.py -q -x 2>&1 | tail -1
timeout 300 python bench.py --no-packed16 --no-cpu --no-e2e --no-johnson --steps 5 > gpurun_out/b.json 2>/dev/null; summ gpurun_out/b.json "int32 cfg2"
timeout 600 python tools/fw_ab.py --n 32768 --deg 64 --dtype f32 --runs 1 2>&1 | tail -1
timeout 1500 python tools/fw_ab.py --n 131072 --deg 256 --dtype f32 --runs 1 > gpurun_out/fw_ab_cfg4_x.json 2>&1; tail -1 gpurun_out/fw_ab_cfg4_x.json
