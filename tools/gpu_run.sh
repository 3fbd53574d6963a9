#!/bin/bash
# One parametrised GPU-box recipe (replaces the round-1 one-off scripts):
#   tools/gpu_run.sh tests [pytest -k expr]   -m gpu tests -> gpurun_out/pytest_gpu.log
#   tools/gpu_run.sh bench [bench.py args]    bench line  -> gpurun_out/bench.json (+ .err)
#   tools/gpu_run.sh ref   [bench.py args]    reference arm -> gpurun_out/ref.json
#   tools/gpu_run.sh cmd '<shell>'            anything else
set -u
mkdir -p gpurun_out
what=$1; shift
case $what in
  tests) python -m pytest tests -m gpu ${PYTEST_X--x} -q ${1:+-k "$1"} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?";
         tail -5 gpurun_out/pytest_gpu.log ;;
  bench) python bench.py "$@" > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?";
         tail -c 600 gpurun_out/bench.json; tail -5 gpurun_out/bench.err ;;
  ref)   python bench.py --impl reference "$@" > gpurun_out/ref.json 2> gpurun_out/ref.err; echo "ref rc=$?";
         tail -c 1500 gpurun_out/ref.json ;;
  cmd)   bash -c "$1" ;;
esac
