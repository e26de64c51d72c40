#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_run.py > gpurun_out/r2_san_racecheck_w1.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_san_racecheck_w1.txt
SAN_GPU_DRAIN=1 SAN_FUSED=0 timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_run.py > gpurun_out/r2_san_racecheck_w1_gpudrain.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_san_racecheck_w1_gpudrain.txt
timeout 1500 compute-sanitizer --tool racecheck --target-processes all --print-limit 20 python -m pytest -q -x tests/test_gpu_multirank.py -k "test_two_ranks_parity and adagrad-False-False-False-False-True" > gpurun_out/r2_san_racecheck_w2.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_san_racecheck_w2.txt
