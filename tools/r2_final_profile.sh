#!/bin/bash
# Round-2 final code on one B200, part 1: smoke, the whole GPU suite, ncu launch lists and
# --set full captures of the top kernels (configs[1], configs[2], FB15k) for profiles/
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2f_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2f_smoke.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q --durations=40 > gpurun_out/r2f_gputests.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2f_gputests.log
bash tools/profile_round.sh criteo_kaggle
bash tools/profile_round.sh avazu
bash tools/profile_round.sh fb15k
ls gpurun_out/prof_*
