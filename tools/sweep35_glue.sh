#!/bin/bash
# Glue variants with the fused lookup: register-cached rows (default) vs re-read (FRUGAL_GLUE_CACHE=0);
# shuffle-broadcast row indices are in both.  Parity of the fused tests first.
timeout 900 python -m pytest tests -m gpu -x -q -k "fused" > gpurun_out/s35_tests.log 2>&1
FRUGAL_GLUE_CACHE=0 timeout 900 python -m pytest tests -m gpu -x -q -k "fused or tiny_100" >> gpurun_out/s35_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/s35_tests.log
for i in 1 2; do
  python bench.py --no-cpu-baseline > gpurun_out/s35_cache_$i.json 2>> gpurun_out/s35.err
  FRUGAL_GLUE_CACHE=0 python bench.py --no-cpu-baseline > gpurun_out/s35_nocache_$i.json 2>> gpurun_out/s35.err
done
python bench.py --no-cpu-baseline --config avazu > gpurun_out/s35_avazu_cache.json 2>> gpurun_out/s35.err
FRUGAL_GLUE_CACHE=0 python bench.py --no-cpu-baseline --config avazu > gpurun_out/s35_avazu_nocache.json 2>> gpurun_out/s35.err
B="python bench.py --steps 40 --warmup 3 --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_dot_model --launch-skip 10 -c 10 --csv \
    --log-file gpurun_out/s35_dm_cache.csv $B > /dev/null 2>&1
FRUGAL_GLUE_CACHE=0 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_dot_model --launch-skip 10 -c 10 --csv \
    --log-file gpurun_out/s35_dm_nocache.csv $B > /dev/null 2>&1
