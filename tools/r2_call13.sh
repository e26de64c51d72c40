#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
timeout 2400 python -m pytest tests -m gpu -q -x --durations=5 -k "not freebase and not avazu and not 100_steps_recorded" > gpurun_out/r2_c13_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c13_tests.log
REPEAT=2 STEPS=300 bash tools/sweep.sh criteo_kaggle "X=default" "FRUGAL_PACK_BLOCKS=40" > gpurun_out/r2_c13_sweep.txt 2>&1
TL_STEPS=80 python tools/timeline.py > gpurun_out/r2_c13_timeline.txt 2>&1
