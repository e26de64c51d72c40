#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
nproc > gpurun_out/r2_c5_nproc.txt; lscpu | head -20 >> gpurun_out/r2_c5_nproc.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2_c5_smoke.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q --durations=30 > gpurun_out/r2_c5_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c5_tests.log
python bench.py > gpurun_out/r2_c5_bench.json 2> gpurun_out/r2_c5_bench.err
REPEAT=1 STEPS=300 bash tools/sweep.sh criteo_kaggle "FRUGAL_FLUSH_THREADS=2" "FRUGAL_FLUSH_THREADS=4" "FRUGAL_FLUSH_THREADS=8" "--drain gpu" > gpurun_out/r2_c5_sweep.txt 2>&1
