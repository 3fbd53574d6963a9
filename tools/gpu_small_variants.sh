#!/bin/bash
# small-n kernel queue variants (tuning): list order + fusion (default), without fusion, the
# 128-kernel's segment order; 1 and 2 CTAs per SM; n = 1024 and 2048
mkdir -p gpurun_out
for n in 1024 2048; do for v in bl bl_nofuse decode; do for c in 1 2; do
  echo "== n=$n queue=$v ctas=$c"
  APSP_SMALL_QUEUE=$v APSP_SMALL_CTAS=$c python tools/fw_ab.py --n $n --deg 8 --dtype i32 --runs 30 --modes small
done; done; done > gpurun_out/small_variants.txt 2>&1
cat gpurun_out/small_variants.txt
