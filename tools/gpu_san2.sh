mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
san() {
  SAN_CASES="$2" timeout 1200 compute-sanitizer --tool $1 --print-limit 10 python tools/san_case.py > gpurun_out/san_$3.log 2>&1
  echo "== $3 ($1, cases '${2:-all}') rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|san_case done|^ok " gpurun_out/san_$3.log | sort | uniq -c
}
san racecheck "barrier,ooc,johnson,boundary" racecheck_barrier
san synccheck "barrier,ooc,johnson,boundary" synccheck_barrier
bash tools/gpu_f32prof.sh
