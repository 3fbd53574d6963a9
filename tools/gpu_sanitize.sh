# compute-sanitizer over tools/san_case.py (every kernel family at small n). memcheck and initcheck
# on all cases; racecheck and synccheck on all cases and on the CTA-barrier-only subset (no mbarrier
# pipelines, which these two tools do not model). Logs -> gpurun_out/san_*.log
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
san() {  # tool, cases, tag
  SAN_CASES="$2" timeout 1200 compute-sanitizer --tool $1 --print-limit 10 python tools/san_case.py > gpurun_out/san_$3.log 2>&1
  echo "== $3 ($1, cases '${2:-all}') rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|san_case done|^ok " gpurun_out/san_$3.log | sort | uniq -c
}
san memcheck "" memcheck
san initcheck "" initcheck
san racecheck "barrier,ooc,johnson,boundary" racecheck_barrier
san synccheck "barrier,ooc,johnson,boundary" synccheck_barrier
san racecheck "dataflow,small" racecheck_dataflow
san synccheck "dataflow" synccheck_dataflow
