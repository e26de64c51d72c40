#!/bin/bash
# session 2, call 4: glue with 8 rows in flight, short-row update ILP, world-1 early host gather (lag rule)
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "pipeline_modes or overlapped_pipeline" > gpurun_out/r2_c28_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c28_tests.log
O=gpurun_out/r2_c28_sweep.txt
sweep() {  # "env..." "bench args"
  env $1 python bench.py --no-cpu-baseline --steps 300 --warmup 20 $2 2>>gpurun_out/r2_c28_err.txt | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1 $2', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), 'frac', round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v})" >> $O 2>&1
}
for i in 1 2; do
  sweep X=1 ""
  sweep FRUGAL_GLUE_UNROLL=1 ""
  sweep FRUGAL_UPDATE_SHORT=0 ""
  sweep "FRUGAL_GLUE_UNROLL=1 FRUGAL_UPDATE_SHORT=0" ""
  sweep FRUGAL_EARLY=1 ""
  sweep "FRUGAL_EARLY=1 FRUGAL_EARLY_BLOCKS=32" ""
  sweep "FRUGAL_EARLY=1 FRUGAL_EARLY_BLOCKS=64" ""
  sweep "FRUGAL_EARLY=1 FRUGAL_EARLY_BLOCKS=32 FRUGAL_EARLY_ROWS=1" ""
done
FRUGAL_EARLY=1 FRUGAL_EARLY_BLOCKS=32 python tools/timeline.py > gpurun_out/r2_c28_timeline_early.txt 2>&1
