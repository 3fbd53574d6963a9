# configs 3 and 4 through the bench's device-timed path (dataflow kernel), single GPU
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/big_build.log 2>&1
timeout 900 python bench.py --workload cfg3_er65536 --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_cfg3.json 2> gpurun_out/bench_cfg3.err; tail -c 400 gpurun_out/bench_cfg3.json; tail -2 gpurun_out/bench_cfg3.err
timeout 1500 python bench.py --workload cfg4_er131072_f32 --steps 1 --warmup 1 --no-e2e --no-cpu --no-johnson > gpurun_out/bench_cfg4.json 2> gpurun_out/bench_cfg4.err; tail -c 400 gpurun_out/bench_cfg4.json; tail -2 gpurun_out/bench_cfg4.err
