#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck / initcheck on the world-1 default path, the GPU
# scatter drain, and the 2-rank test (both ranks on one GPU); summaries -> gpurun_out/r2_san_*.txt
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
CS=compute-sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 $CS --tool $tool --print-limit 20 python tools/sanitize_run.py > gpurun_out/r2_san_${tool}_w1.txt 2>&1
  echo "rc=$?" >> gpurun_out/r2_san_${tool}_w1.txt
done
SAN_GPU_DRAIN=1 SAN_FUSED=0 timeout 900 $CS --tool memcheck --print-limit 20 python tools/sanitize_run.py > gpurun_out/r2_san_memcheck_w1_gpudrain.txt 2>&1
echo "rc=$?" >> gpurun_out/r2_san_memcheck_w1_gpudrain.txt
for tool in memcheck racecheck synccheck; do
  timeout 1500 $CS --tool $tool --target-processes all --print-limit 20 python -m pytest -q -x tests/test_gpu_multirank.py -k "test_two_ranks_parity and adagrad-False-False-False-False-True" > gpurun_out/r2_san_${tool}_w2.txt 2>&1
  echo "rc=$?" >> gpurun_out/r2_san_${tool}_w2.txt
done
