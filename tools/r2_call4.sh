#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
timeout 300 python bench.py --drain host --no-cpu-baseline --steps 100 --warmup 10 > gpurun_out/r2_c4_host.json 2> gpurun_out/r2_c4_host.err
echo "host rc=$?" >> gpurun_out/r2_c4_host.err
timeout 900 python -m pytest tests -m gpu -q -x -k "tiny_100 or fused_lookup or overlapped_pipeline_tiny or dims or host_flush_recorded" > gpurun_out/r2_c4_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c4_tests.log
REPEAT=2 STEPS=300 bash tools/sweep.sh criteo_kaggle "X=default" "FRUGAL_GLUE_RG=0" > gpurun_out/r2_c4_sweep.txt 2>&1
REPEAT=1 STEPS=300 bash tools/sweep.sh avazu "X=default" "FRUGAL_GLUE_RG=0" >> gpurun_out/r2_c4_sweep.txt 2>&1
