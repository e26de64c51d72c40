#!/bin/bash
# Shuffle-broadcast row indices in the re-read (uncached) fused glue too: parity, then Avazu x3 + Criteo
# (compare with sweep 35/36 and r1_bench_avazu.json: 37.4-37.6 M before).
timeout 900 python -m pytest tests -m gpu -x -q -k "fused or pipeline_modes or tiny_100" > gpurun_out/s37_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/s37_tests.log
for i in 1 2 3; do
  python bench.py --no-cpu-baseline --config avazu > gpurun_out/s37_avazu_$i.json 2>> gpurun_out/s37.err
done
python bench.py --no-cpu-baseline > gpurun_out/s37_criteo.json 2>> gpurun_out/s37.err
