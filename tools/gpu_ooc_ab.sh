#!/bin/bash
# out-of-core timing: every band streamed (the paper's setting) and with resident bands
mkdir -p gpurun_out
{
python tools/ooc_ab.py --n 16384 --block 2048 --stream-all --runs 2
python tools/ooc_ab.py --n 16384 --block 4096 --stream-all --runs 2
python tools/ooc_ab.py --n 32768 --block 4096 --stream-all --runs 1
python tools/ooc_ab.py --n 32768 --block 4096 --stream-all --runs 1 --world 2
} > gpurun_out/ooc_ab.txt 2>&1
cat gpurun_out/ooc_ab.txt
