# fp32: ncu of the dataflow kernel vs a per-phase phase-3 launch (n=16384 ER deg 64)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:fw_dataflow_kernel -c 1 -o gpurun_out/f32_df python tools/profile_fw.py --er 16384 --deg 64 --dtype f32 --dataflow --runs 1 > gpurun_out/ncu_f32_df.log 2>&1; tail -1 gpurun_out/ncu_f32_df.log
timeout 900 ncu --set full --import-source on --clock-control none -k regex:minplus --launch-skip 200 -c 3 -o gpurun_out/f32_pp python tools/profile_fw.py --er 16384 --deg 64 --dtype f32 --legacy --runs 1 > gpurun_out/ncu_f32_pp.log 2>&1; tail -1 gpurun_out/ncu_f32_pp.log
timeout 900 ncu --set full --import-source on --clock-control none -k regex:fw_dataflow_kernel -c 1 -o gpurun_out/i32_df python tools/profile_fw.py --runs 1 > gpurun_out/ncu_i32_df.log 2>&1; tail -1 gpurun_out/ncu_i32_df.log
