mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python tools/fw_ab.py --n 32768 --deg 64 --dtype f32 --runs 1 2>&1 | tail -1
timeout 900 python tools/fw_ab.py --n 65536 --deg 16 --dtype i32 --runs 1 --modes dataflow 2>&1 | tail -1
APSP_NVCC_EXTRA="-DDF_INLINE" python -c "
import importlib.util
spec=importlib.util.spec_from_file_location('b','paper_conf_ipps_xia0ar22_b200/_build.py'); b=importlib.util.module_from_spec(spec); spec.loader.exec_module(b); b.build_lib(force=True)" > /dev/null
echo "== DF_INLINE"
timeout 900 python tools/fw_ab.py --n 32768 --deg 64 --dtype f32 --runs 1 --modes dataflow 2>&1 | tail -1
timeout 600 python tools/fw_ab.py --n 16384 --deg 8 --dtype i32 --runs 2 --modes dataflow 2>&1 | tail -1
