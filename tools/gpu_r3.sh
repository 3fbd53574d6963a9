mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -c 300 gpurun_out/bench.json; echo
timeout 900 python tools/fw_ab.py --n 32768 --deg 256 --dtype f32 > gpurun_out/fw_ab_f32_v3.json 2>&1; cat gpurun_out/fw_ab_f32_v3.json
timeout 900 python tools/fw_ab.py --n 131072 --deg 8 --dtype i32 --runs 1 --modes dataflow > gpurun_out/fw_ab_i32_131072.json 2>&1; cat gpurun_out/fw_ab_i32_131072.json
timeout 1500 python bench.py --workload cfg4_er131072_f32 --steps 1 --warmup 1 --no-e2e --no-cpu --no-johnson > gpurun_out/bench_cfg4.json 2> gpurun_out/bench_cfg4.err; tail -c 300 gpurun_out/bench_cfg4.json; tail -2 gpurun_out/bench_cfg4.err
