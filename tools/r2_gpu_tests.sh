#!/bin/bash
# GPU parity suite + smoke + headline bench line on one B200 (round 2)
cd "${GRAFT_REPO_ROOT:-.}"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2_smoke.log 2>&1
timeout ${TEST_TIMEOUT:-2400} python -m pytest tests -m gpu -q --durations=40 ${PYTEST_ARGS} > gpurun_out/r2_gputests.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_gputests.log
python bench.py > gpurun_out/r2_bench.json 2> gpurun_out/r2_bench.err
tail -3 gpurun_out/r2_gputests.log
