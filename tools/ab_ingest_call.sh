#!/bin/bash
# A/B on one box: ingest copy + part A after the caller's prior work only (new) vs after this
# step's scheduler too (previous), alternating, configs[1]; then the parity subset on the new code
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null
rm -rf /tmp/varB && mkdir -p /tmp/varB && cp -r paper_conf_asplos_xiezggl25_b200 include bench.py oracle __graft_entry__.py MEASURED_PEAKS.json profiles /tmp/varB/ 2>/dev/null
cp gpurun_ab/runtime_prev.cu /tmp/varB/paper_conf_asplos_xiezggl25_b200/csrc/runtime.cu
(cd /tmp/varB && python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null)
O=gpurun_out/ab_ingest_call.txt; rm -f $O
run() { (cd $1 && python bench.py --no-cpu-baseline --steps 300 --warmup 20 $3 2>/dev/null) | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$2 $3', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v})" >> $O; }
for i in 1 2 3; do run . A_new; run /tmp/varB B_prev; done
run . A_new "--config avazu"; run /tmp/varB B_prev "--config avazu"
python tools/timeline.py > gpurun_out/ab_timeline_new.txt 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -m gpu -q -x -k "tiny or overlapped or pipeline_modes or criteo_kaggle_100 or two_ranks_parity" > gpurun_out/ab_tests.log 2>&1
echo "rc=$?" >> gpurun_out/ab_tests.log
