# Config 5 (n=262144 int32, 275 GB) out of core on one B200, every row certified.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/cfg5_build.log 2>&1
free -g > gpurun_out/cfg5_mem.txt
nvidia-smi --query-gpu=timestamp,clocks.sm,clocks.max.sm,power.draw,clocks_throttle_reasons.active --format=csv -l 15 > gpurun_out/cfg5_clocks.csv 2>&1 &
SMI=$!
timeout 3300 python tests/perf/ooc_scale.py --certify --rows 64 > gpurun_out/cfg5_ooc.json 2> gpurun_out/cfg5_ooc.err
echo "rc=$?"
kill $SMI
tail -c 3000 gpurun_out/cfg5_ooc.json; tail -5 gpurun_out/cfg5_ooc.err
