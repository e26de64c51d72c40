#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
timeout 1500 python -m pytest tests -m gpu -q --durations=5 -k "contents_every_step" > gpurun_out/r2_c11_contents.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x --durations=5 -k "not contents_every_step" > gpurun_out/r2_c11_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c11_tests.log
REPEAT=2 STEPS=300 bash tools/sweep.sh criteo_kaggle "X=default" "FRUGAL_URGENT_SIDE=0" > gpurun_out/r2_c11_sweep.txt 2>&1
python bench.py > gpurun_out/r2_c11_bench.json 2> gpurun_out/r2_c11_bench.err
