# bench (default) + Johnson ncu capture + launch list of the bench
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -c 1500 gpurun_out/bench.json; echo; tail -3 gpurun_out/bench.err
timeout 600 ncu --set full --import-source on --clock-control none -k regex:mssp --launch-skip 1 -c 1 -o gpurun_out/jn_full python tools/profile_jn.py > gpurun_out/ncu_jn.log 2>&1; tail -2 gpurun_out/ncu_jn.log
