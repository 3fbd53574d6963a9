# Johnson (batched Near-Far) + selector tests, then default-config benches on configs 2 and 3.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/jn_build.log 2>&1 || tail -20 gpurun_out/jn_build.log
timeout 900 python -m pytest tests/test_gpu_johnson.py tests/test_gpu_select.py -q -x > gpurun_out/jn_pytest.log 2>&1; tail -15 gpurun_out/jn_pytest.log
timeout 900 python tests/perf/johnson_bench.py --workload cfg2_grid16384 --steps 5 --warmup 2 --deltas 0 150 300 --fw > gpurun_out/jn_bench_cfg2.json 2> gpurun_out/jn_bench.err; tail -c 300 gpurun_out/jn_bench_cfg2.json; tail -3 gpurun_out/jn_bench.err
timeout 1200 python tests/perf/johnson_bench.py --workload cfg3_er65536 --deltas 0 8 20 --steps 2 > gpurun_out/jn_bench_cfg3.json 2>> gpurun_out/jn_bench.err; tail -c 300 gpurun_out/jn_bench_cfg3.json; tail -3 gpurun_out/jn_bench.err
