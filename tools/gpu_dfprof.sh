mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
APSP_DF_PROFILE=1 python tools/profile_fw.py --runs 2 2>&1 | grep "\[df\]"
APSP_DF_PROFILE=1 python tools/profile_fw.py --workload cfg3_er65536 --runs 1 2>&1 | grep "\[df\]"
