mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:fw_dataflow16 -c 1 -o gpurun_out/df16i_full python tools/profile_fw.py --packed16 --runs 1 > gpurun_out/ncu16i.log 2>&1
tail -1 gpurun_out/ncu16i.log
