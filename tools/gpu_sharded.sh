mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_sharded.py -q -x > gpurun_out/pytest_sharded.log 2>&1; tail -25 gpurun_out/pytest_sharded.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dataflow.py -q -x 2>&1 | tail -3
timeout 600 python tools/fw_ab.py --n 16384 --deg 8 --dtype i32 --runs 2 --modes dataflow 2>&1 | tail -1
timeout 600 python tools/vr_bench.py 2>&1 | tail -5
