#!/bin/bash
# (written when the fused lookup was opt-in; now the default, so base = --no-fused-lookup)
# Fused lookup (glue reads gathered distinct rows via inv; no expand): parity, then A/B bench.
timeout 900 python -m pytest tests -m gpu -x -q -k "fused or pipeline_modes" > gpurun_out/fused_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/fused_tests.log
for i in 1 2; do
  python bench.py --no-cpu-baseline --no-fused-lookup > gpurun_out/s32_base_$i.json 2>> gpurun_out/s32.err
  python bench.py --no-cpu-baseline > gpurun_out/s32_fused_$i.json 2>> gpurun_out/s32.err
done
python bench.py --no-cpu-baseline --config avazu --no-fused-lookup > gpurun_out/s32_avazu_base.json 2>> gpurun_out/s32.err
python bench.py --no-cpu-baseline --config avazu > gpurun_out/s32_avazu_fused.json 2>> gpurun_out/s32.err
