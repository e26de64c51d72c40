#!/bin/bash
# host-flush drain + one-launch update kernel: parity, then A/B bench lines (configs[1])
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
timeout 1200 python -m pytest tests -m gpu -q -x -k "host_flush or tiny_100 or long_segments or overlapped_pipeline or dims or fused_lookup_shapes or kg_transe or dynamic_cache" > gpurun_out/r2_c3_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c3_tests.log
tail -3 gpurun_out/r2_c3_tests.log
REPEAT=2 STEPS=300 bash tools/sweep.sh criteo_kaggle "X=default" "--drain host" "FRUGAL_UPDATE1=0" "--drain host FRUGAL_FLUSH_THREADS=8" > gpurun_out/r2_c3_sweep.txt 2>&1
cat gpurun_out/r2_c3_sweep.txt
