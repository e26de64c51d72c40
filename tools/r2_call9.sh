#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
timeout 1500 python -m pytest tests -m gpu -q -x --durations=5 -k "not freebase and not avazu and not 100_steps_recorded" > gpurun_out/r2_c9_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c9_tests.log
python tools/host_profile.py > gpurun_out/r2_c9_host.txt 2>&1
TL_STEPS=80 python tools/timeline.py > gpurun_out/r2_c9_timeline.txt 2>&1
python bench.py --no-cpu-baseline > gpurun_out/r2_c9_bench.json 2> gpurun_out/r2_c9_bench.err
python bench.py --no-cpu-baseline --config avazu > gpurun_out/r2_c9_bench_avazu.json 2>> gpurun_out/r2_c9_bench.err
