# flakiness check: the GPU suite three times in a row, plus memcheck on the final code
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for i in 1 2 3; do timeout 1200 python -m pytest tests -m gpu -q -p no:randomly > gpurun_out/pytest_gpu_$i.log 2>&1; tail -1 gpurun_out/pytest_gpu_$i.log; done
SAN_CASES="" timeout 1200 compute-sanitizer --tool memcheck --print-limit 10 python tools/san_case.py > gpurun_out/san_memcheck_final.log 2>&1; echo "memcheck rc=$?"; grep -E "ERROR SUMMARY|san_case done" gpurun_out/san_memcheck_final.log
