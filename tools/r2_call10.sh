#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
timeout 1500 python -m pytest tests -m gpu -q -x --durations=5 -k "not freebase and not avazu and not multirank" > gpurun_out/r2_c10_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c10_tests.log
TL_STEPS=80 python tools/timeline.py > gpurun_out/r2_c10_timeline.txt 2>&1
REPEAT=2 STEPS=300 bash tools/sweep.sh criteo_kaggle "X=default" "FRUGAL_URGENT_SIDE=0" > gpurun_out/r2_c10_sweep.txt 2>&1
