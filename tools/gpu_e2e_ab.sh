mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
(cd _ab/old && python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1)
summ() { python -c "
import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); e=d['e2e']
print(sys.argv[2], 'e2e', e['value'], e.get('ms_parts_each_step'), e.get('serial',{}).get('ms_parts_each_step'))" $1 $2; }
(cd _ab/old && timeout 600 python bench.py --no-cpu --no-johnson --no-packed16 --steps 3 > ../old.json 2>/dev/null); summ _ab/old.json old
timeout 600 python bench.py --no-cpu --no-johnson --no-packed16 --steps 3 > _ab/new.json 2>/dev/null; summ _ab/new.json new
(cd _ab/old && timeout 600 python bench.py --no-cpu --no-johnson --no-packed16 --steps 3 > ../old2.json 2>/dev/null); summ _ab/old2.json old2
