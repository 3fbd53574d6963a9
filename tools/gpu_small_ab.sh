#!/bin/bash
# small-n kernel A/B (64-tile vs 128-tile dataflow vs per-phase) at n = 1024 .. 4096
mkdir -p gpurun_out
for n in 1024 2048 3072 4096; do
  python tools/fw_ab.py --n $n --deg 8 --dtype i32 --runs 20 --modes small dataflow per_phase
done > gpurun_out/small_ab.txt 2>&1
for c in 2 3; do APSP_SMALL_CTAS=$c python tools/fw_ab.py --n 1024 --deg 8 --dtype i32 --runs 20 --modes small; done >> gpurun_out/small_ab.txt 2>&1
python tools/fw_ab.py --n 1024 --deg 64 --dtype f32 --runs 20 --modes small dataflow per_phase >> gpurun_out/small_ab.txt 2>&1
cat gpurun_out/small_ab.txt
