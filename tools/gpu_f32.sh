# fp32 min-plus: micro peaks (incl. FADD2+FMNMX3 broadcast form), FW A/B at n=32768/65536, OOC phase-3 ncu
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/f32_build.log 2>&1 || tail -20 gpurun_out/f32_build.log
./build/dpx_peak > gpurun_out/dpx_peak2.json; cat gpurun_out/dpx_peak2.json
timeout 600 python tools/fw_ab.py --n 32768 --deg 256 --dtype f32 > gpurun_out/fw_ab_f32_v2.json 2>&1; cat gpurun_out/fw_ab_f32_v2.json
timeout 900 python tools/fw_ab.py --n 65536 --deg 16 --dtype f32 --runs 1 > gpurun_out/fw_ab_f32_65536.json 2>&1; cat gpurun_out/fw_ab_f32_65536.json
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dataflow.py tests/test_gpu_johnson.py -q -x > gpurun_out/f32_pytest.log 2>&1; tail -3 gpurun_out/f32_pytest.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:minplus --csv --log-file gpurun_out/ooc_launches.csv python tools/profile_fw.py --ooc-block 4096 --runs 1 > /dev/null 2>&1
SKIP=$(python - <<'PY'
import csv, io
rows = [r for r in csv.DictReader(io.StringIO(''.join(l for l in open('gpurun_out/ooc_launches.csv') if not l.startswith('=='))))]
idx = [i for i, r in enumerate(rows) if float(r['Metric Value']) > 5e6]
print(idx[0] if idx else 0)
PY
)
echo "skip=$SKIP"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:minplus --launch-skip $SKIP -c 1 -o gpurun_out/ooc_p3 python tools/profile_fw.py --ooc-block 4096 --runs 1 > gpurun_out/ncu_ooc.log 2>&1; tail -1 gpurun_out/ncu_ooc.log
