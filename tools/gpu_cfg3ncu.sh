mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:fw_dataflow -c 1 --csv --log-file gpurun_out/cfg3_ncu.csv python tools/profile_fw.py --workload cfg3_er65536 --runs 1 > gpurun_out/cfg3_ncu.log 2>&1
tail -2 gpurun_out/cfg3_ncu.log; grep -v "^==" gpurun_out/cfg3_ncu.csv | cut -d, -f12- | tail -6
