mkdir -p gpurun_out
out=gpurun_out/small_split.txt
{ timeout 600 python -m pytest tests/test_gpu_small.py tests/test_gpu_golden.py -q -x 2>&1 | tail -5
  for rep in 1 2; do for s in 1 2 4; do for n in 1024 2048; do
    echo "== split=$s n=$n"; APSP_SMALL_SPLIT=$s timeout 120 python tools/fw_ab.py --n $n --deg 8 --dtype i32 --runs 30 --modes small
  done; done; done
  for s in 1 2 4; do echo "== split=$s profile"; APSP_SMALL_SPLIT=$s APSP_SMALL_PROFILE=1 timeout 120 python tools/fw_ab.py --n 1024 --deg 8 --dtype i32 --runs 3 --modes small 2>&1 | grep small; done
} > $out 2>&1
cat $out | cut -c1-400
