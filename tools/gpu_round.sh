# Full GPU pass (gpurun): tests, smoke, bench (default workload), ncu launch list + one --set full capture.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; tail -1 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -c 400 gpurun_out/bench.json; echo
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-packed16 > gpurun_out/bench_ncu.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:fw_dataflow --launch-skip 1 -c 1 -o gpurun_out/df_full python tools/profile_fw.py > gpurun_out/ncu_full.log 2>&1
tail -1 gpurun_out/ncu_full.log
