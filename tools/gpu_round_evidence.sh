#!/bin/bash
# Round evidence on one B200: -m gpu tests, smoke, the driver's bench command + reference arm, the
# ncu launch list of a short bench run, ncu --set full of the dominant kernel (the two-round
# dataflow kernel at n = 16384) and its DRAM traffic at config 3. Outputs under gpurun_out/.
mkdir -p gpurun_out
R=${ROUND:-r02}
tools/gpu_run.sh tests
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
tools/gpu_run.sh bench --steps 20 --warmup 5
tools/gpu_run.sh ref --steps 20 --warmup 5
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv \
  --log-file gpurun_out/${R}_launches_bench.csv python bench.py --steps 2 --warmup 1 > gpurun_out/${R}_bench_under_ncu.log 2>&1
echo "launch list rc=$?"
APSP_DF_PAIR=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:fw_dataflow_kernel --launch-skip 1 -c 1 \
  -o gpurun_out/${R}_ncu_dataflow_pair_n16384 -f python tools/profile_fw.py --er 16384 --deg 8 --runs 2 > /dev/null 2>&1
echo "ncu full rc=$?"
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active \
  --clock-control none -k regex:fw_dataflow_kernel -c 1 --csv --log-file gpurun_out/${R}_ncu_cfg3_pair_traffic.csv \
  python tools/profile_fw.py --workload cfg3_er65536 --runs 1 > /dev/null 2>&1
echo "ncu cfg3 rc=$?"
