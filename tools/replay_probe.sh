#!/bin/bash
# exact host-row replay (profiles/r1_exact_replay.txt): build tools/layout_probe2 first
# (nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/layout_probe2 tools/layout_probe2.cu)
DUMP_STEPS=100 python tools/dump_lists.py > gpurun_out/dump8.txt 2>&1
python tools/lay_remap.py >> gpurun_out/dump8.txt 2>&1
./tools/layout_probe2 > gpurun_out/layout_probe8.txt 2>&1
