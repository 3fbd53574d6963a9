# ncu --set full of the packed16 dataflow kernel on cfg2 (one launch), with source counters.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:fw_dataflow16 -c 1 -o gpurun_out/df16_full python tools/profile_fw.py --packed16 --runs 1 > gpurun_out/ncu16.log 2>&1
tail -2 gpurun_out/ncu16.log
