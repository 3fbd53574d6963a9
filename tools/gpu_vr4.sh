mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python tools/vr_bench.py --n 65536 --worlds 1 8 --runs 1 2>&1 | tail -1
