mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/jn_build.log 2>&1 || tail -20 gpurun_out/jn_build.log
timeout 900 python tests/perf/johnson_bench.py --workload cfg2_grid16384 --steps 6 --warmup 3 --deltas 200 400 --env "APSP_JN_THREADS=256" "" "APSP_JN_THREADS=256,APSP_JN_CTAS_PER_SM=4" "APSP_JN_SMEM_DIST=1,APSP_JN_THREADS=256" "APSP_JN_THREADS=256" > gpurun_out/jn_bench_cfg2.json 2> gpurun_out/jn_bench.err; tail -3 gpurun_out/jn_bench.err
nvidia-smi --query-gpu=clocks.sm,clocks_throttle_reasons.active --format=csv
