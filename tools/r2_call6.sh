#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
timeout 900 python -m pytest tests -m gpu -q -x -k "own_ids or tiny_100 or gpu_drain_recorded or flushing_threads or overlapped_pipeline_tiny" > gpurun_out/r2_c6_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c6_tests.log
TL_STEPS=80 python tools/timeline.py > gpurun_out/r2_c6_timeline.txt 2>&1
REPEAT=2 STEPS=300 bash tools/sweep.sh criteo_kaggle "X=default" "FRUGAL_PACK_BLOCKS=40" "FRUGAL_PACK_BLOCKS=80" > gpurun_out/r2_c6_sweep.txt 2>&1
