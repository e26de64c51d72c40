#!/bin/bash
# Criteo (d 32) glue variant with the fused lookup, longer alternating A/B: cached (auto) vs re-read.
for i in 1 2 3 4; do
  python bench.py --no-cpu-baseline --steps 400 > gpurun_out/s36_cache_$i.json 2>> gpurun_out/s36.err
  FRUGAL_GLUE_CACHE=0 python bench.py --no-cpu-baseline --steps 400 > gpurun_out/s36_nocache_$i.json 2>> gpurun_out/s36.err
done
