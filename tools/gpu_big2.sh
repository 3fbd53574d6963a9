# bench lines for configs 3 and 4 on one GPU with the final code
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python bench.py --workload cfg3_er65536 --steps 3 --warmup 3 --no-johnson > gpurun_out/bench_cfg3.json 2> gpurun_out/bench_cfg3.err; tail -c 300 gpurun_out/bench_cfg3.json; echo
timeout 2700 python bench.py --workload cfg4_er131072_f32 --steps 3 --warmup 3 --no-johnson --no-e2e > gpurun_out/bench_cfg4.json 2> gpurun_out/bench_cfg4.err; tail -c 300 gpurun_out/bench_cfg4.json; echo
