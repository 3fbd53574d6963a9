mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/ck_build.log 2>&1 || tail -20 gpurun_out/ck_build.log
timeout 900 python -m pytest tests/test_gpu_checkpoint.py tests/test_gpu_johnson.py tests/test_gpu_ooc.py tests/test_gpu_parity.py -q -x > gpurun_out/ck_pytest.log 2>&1; tail -15 gpurun_out/ck_pytest.log
