# de-phase the two CTAs of an SM (APSP_DF_STAGGER: cycles the second half of the grid waits before its first task)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], '%.4e'%d['value'], '%.2f ms'%d['ms_per_step'], 'frac %.4f'%r['frac'])" $1 "$2"; }
for rep in 1 2; do
for st in 0 8000 32000 64000; do
  APSP_DF_STAGGER=$st timeout 300 python bench.py --no-packed16 --no-cpu --no-e2e --no-johnson --steps 5 > gpurun_out/b.json 2>/dev/null; summ gpurun_out/b.json "stagger=$st"
done
done
APSP_DF_STAGGER=32000 APSP_DF_PROFILE=1 python tools/profile_fw.py --runs 2 2>&1 | grep "\[df\]"
