#!/bin/bash
# A/B timing recipes for one B200 (device time via tools/fw_ab.py / tools/ooc_ab.py), output in
# gpurun_out/ab_<what>.txt:
#   tools/gpu_ab.sh small   64-tile small-n kernel vs the 128-tile kernels, n = 1024 .. 4096, CTAs per SM
#   tools/gpu_ab.sh close   small-n phase 1: deferred-bulk closure (default) vs one barrier per step
#   tools/gpu_ab.sh pair    two-round (pair) queue vs one-round queue, int32 n = 16384 / 32768 / 65536, fp32
#   tools/gpu_ab.sh ooc     out of core, every band streamed (n = 16384 / 32768, 1 and 2 virtual ranks)
#   tools/gpu_ab.sh split   small-n chain panel tiles in 1 / 2 / 4 parts (APSP_SMALL_SPLIT), n = 1024 / 2048
#   tools/gpu_ab.sh exact   int32 engine vs exact_f32 (R25) at n = 16384 / 65536
#   tools/gpu_ab.sh variant NAME [DTYPE]  default build vs build/var_NAME (tools/build_variant.py), dataflow
#                           kernel, n = 16384 / 32768, alternating twice
mkdir -p gpurun_out
what=$1
out=gpurun_out/ab_$what.txt
case $what in
  small)
    { for n in 1024 1536 2048 3072 4096; do
        echo "== n=$n"; python tools/fw_ab.py --n $n --deg 8 --dtype i32 --runs 20 --modes small dataflow per_phase
      done
      for c in 1 2 3; do echo "== n=1024 ctas=$c"; APSP_SMALL_CTAS=$c python tools/fw_ab.py --n 1024 --deg 8 --dtype i32 --runs 20 --modes small; done
      echo "== n=1024 profile"; APSP_SMALL_PROFILE=1 python tools/fw_ab.py --n 1024 --deg 8 --dtype i32 --runs 3 --modes small
    } > $out 2>&1 ;;
  close)
    { for n in 1024 1536 2048; do for v in 0 1 0 1; do
        echo "== close_v=$v n=$n"; APSP_SMALL_CLOSE=$v python tools/fw_ab.py --n $n --deg 8 --dtype i32 --runs 20 --modes small
      done; done
      for v in 0 1; do echo "== close_v=$v profile"; APSP_SMALL_CLOSE=$v APSP_SMALL_PROFILE=1 python tools/fw_ab.py --n 1024 --deg 8 --dtype i32 --runs 3 --modes small; done
    } > $out 2>&1 ;;
  pair)
    { for n in 16384 32768 65536; do
        r=3; d=4; [ $n -gt 16384 ] && r=2; [ $n -gt 32768 ] && r=1 && d=16
        for p in 0 1; do echo "== pair=$p n=$n"; APSP_DF_PAIR=$p python tools/fw_ab.py --n $n --deg $d --dtype i32 --runs $r --modes dataflow; done
      done
      for p in 0 1; do echo "== pair=$p f32 n=32768"; APSP_DF_PAIR=$p python tools/fw_ab.py --n 32768 --deg 64 --dtype f32 --runs 2 --modes dataflow; done
    } > $out 2>&1 ;;
  ooc)
    { python tools/ooc_ab.py --n 16384 --block 2048 --stream-all --runs 2
      python tools/ooc_ab.py --n 16384 --block 4096 --stream-all --runs 2
      python tools/ooc_ab.py --n 32768 --block 4096 --stream-all --runs 1
      python tools/ooc_ab.py --n 32768 --block 4096 --stream-all --runs 1 --world 2
    } > $out 2>&1 ;;
  split)
    { timeout 600 python -m pytest tests/test_gpu_small.py -q -x 2>&1 | tail -3
      for rep in 1 2; do for s in 1 2 4; do for n in 1024 2048; do
        echo "== split=$s n=$n"; APSP_SMALL_SPLIT=$s timeout 120 python tools/fw_ab.py --n $n --deg 8 --dtype i32 --runs 30 --modes small
      done; done; done
      for s in 1 2 4; do echo "== split=$s profile"
        APSP_SMALL_SPLIT=$s APSP_SMALL_PROFILE=1 timeout 120 python tools/fw_ab.py --n 1024 --deg 8 --dtype i32 --runs 3 --modes small
      done
    } > $out 2>&1 ;;
  exact)
    { for n in 16384 65536; do for x in "" "--exact-f32"; do
        echo "== n=$n $x"; timeout 300 python tools/fw_ab.py --n $n --deg 16 --dtype i32 --runs 2 --modes dataflow $x
      done; done
    } > $out 2>&1 ;;
  variant)
    v=$2; dt=${3:-f32}; out=gpurun_out/ab_variant_${v}_${dt}.txt
    { for rep in 1 2; do for n in 16384 32768; do
        r=5; [ $n -gt 16384 ] && r=2
        echo "== default n=$n"; timeout 300 python tools/fw_ab.py --n $n --deg 64 --dtype $dt --runs $r --modes dataflow
        echo "== $v n=$n"; (cd build/var_$v && timeout 300 python tools/fw_ab.py --n $n --deg 64 --dtype $dt --runs $r --modes dataflow)
      done; done
    } > $out 2>&1 ;;
  *) echo "usage: tools/gpu_ab.sh small|close|pair|ooc|split|exact|variant"; exit 2 ;;
esac
cat $out | grep -vE "^\s*$" | tail -40
