#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
timeout 1500 python -m pytest tests -m gpu -q -x --durations=10 > gpurun_out/r2_c8_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c8_tests.log
python tools/host_profile.py > gpurun_out/r2_c8_host.txt 2>&1
FRUGAL_GRAPHS=0 python tools/host_profile.py >> gpurun_out/r2_c8_host.txt 2>&1
python bench.py > gpurun_out/r2_c8_bench.json 2> gpurun_out/r2_c8_bench.err
FRUGAL_GRAPHS=0 python bench.py --no-cpu-baseline > gpurun_out/r2_c8_bench_nograph.json 2>> gpurun_out/r2_c8_bench.err
