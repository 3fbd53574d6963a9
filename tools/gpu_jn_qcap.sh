mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/jn_build.log 2>&1 || tail -20 gpurun_out/jn_build.log
timeout 900 python -m pytest tests/test_gpu_johnson.py tests/test_gpu_select.py -q -x > gpurun_out/jn_pytest.log 2>&1; tail -5 gpurun_out/jn_pytest.log
timeout 900 python tests/perf/johnson_bench.py --workload cfg2_grid16384 --steps 5 --warmup 2 --env "" "APSP_JN_QCAP=0" "APSP_JN_QCAP=256" > gpurun_out/jn_bench_cfg2.json 2> gpurun_out/jn_bench.err; tail -3 gpurun_out/jn_bench.err
timeout 1200 python tests/perf/johnson_bench.py --workload cfg3_er65536 --steps 2 --env "" "APSP_JN_QCAP=0" > gpurun_out/jn_bench_cfg3.json 2>> gpurun_out/jn_bench.err; tail -3 gpurun_out/jn_bench.err
timeout 600 ncu --set full --import-source on --clock-control none -k regex:mssp --launch-skip 1 -c 1 -o gpurun_out/jn_full python tools/profile_jn.py > gpurun_out/ncu_jn.log 2>&1; tail -1 gpurun_out/ncu_jn.log
timeout 900 ncu --set full --import-source on --clock-control none -k regex:minplus --launch-skip 40 -c 1 -o gpurun_out/ooc_p3 python tools/profile_fw.py --ooc-block 4096 --runs 1 > gpurun_out/ncu_ooc.log 2>&1; tail -1 gpurun_out/ncu_ooc.log
timeout 600 python tools/fw_ab.py --n 32768 --deg 256 --dtype f32 > gpurun_out/fw_ab_f32.json 2>&1; cat gpurun_out/fw_ab_f32.json
timeout 600 python tools/fw_ab.py --n 32768 --deg 16 --dtype i32 > gpurun_out/fw_ab_i32.json 2>&1; cat gpurun_out/fw_ab_i32.json
