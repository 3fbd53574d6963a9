mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_sharded.py -q -x 2>&1 | tail -1
timeout 900 python tools/vr_bench.py --n 16384 --worlds 1 2 4 8 2>&1 | tail -1
timeout 900 python tools/vr_bench.py --n 32768 --worlds 2 2>&1 | tail -1
