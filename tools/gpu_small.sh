mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], '%.4e'%d['value'], '%.3f ms'%d['ms_per_step'], 'frac %.4f'%r['frac'])" $1 "$2"; }
for wl in cfg1_er1024; do
  timeout 300 python bench.py --workload $wl --no-packed16 --no-cpu --no-e2e --no-johnson --steps 20 > gpurun_out/b.json 2>/dev/null; summ gpurun_out/b.json "$wl dataflow"
  timeout 300 python bench.py --workload $wl --no-packed16 --no-cpu --no-e2e --no-johnson --steps 20 --legacy > gpurun_out/b.json 2>/dev/null; summ gpurun_out/b.json "$wl per-phase"
  timeout 300 python bench.py --workload $wl --no-cpu --no-e2e --no-johnson --steps 20 --packed16 > gpurun_out/b.json 2>/dev/null; summ gpurun_out/b.json "$wl packed16"
done
APSP_DF_PROFILE=1 python tools/profile_fw.py --workload cfg1_er1024 --runs 2 2>&1 | grep "\[df\]"
