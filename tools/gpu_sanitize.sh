# compute-sanitizer over tools/san_case.py (every kernel family at small n): memcheck, racecheck,
# synccheck, initcheck. Summaries -> gpurun_out/san_*.log
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  SAN_N=${SAN_N:-300} timeout 1200 compute-sanitizer --tool $tool --target-processes all --print-limit 20 python tools/san_case.py > gpurun_out/san_$tool.log 2>&1
  echo "== $tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|san_case done|Error|error" gpurun_out/san_$tool.log | sort | uniq -c | head -8
done
