mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python -m pytest tests/test_gpu_dataflow.py tests/test_gpu_sharded.py -q -x 2>&1 | tail -1
timeout 1500 python tools/fw_ab.py --n 131072 --deg 256 --dtype f32 --runs 1 > gpurun_out/fw_ab_cfg4.json 2>&1; tail -1 gpurun_out/fw_ab_cfg4.json
