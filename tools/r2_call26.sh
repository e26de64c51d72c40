#!/bin/bash
# session 2, call 2: gather with R rows in flight (FRUGAL_GATHER_ROWS) x grid, sampled phase timers
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
O=gpurun_out/r2_c26_sweep.txt
sweep() {  # "env..." "bench args"
  env $1 python bench.py --no-cpu-baseline --steps 300 --warmup 20 $2 2>>gpurun_out/r2_c26_err.txt | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1 $2', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), 'frac', round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v}, d['phase_timers'])" >> $O 2>&1
}
for i in 1 2; do
  sweep X=1 ""
  sweep X=1 "--timer-every 8"
  sweep FRUGAL_GATHER_ROWS=2 ""
  sweep FRUGAL_GATHER_ROWS=4 ""
  sweep "FRUGAL_GATHER_ROWS=4 FRUGAL_GATHER_BLOCKS=148" ""
  sweep "FRUGAL_GATHER_ROWS=4 FRUGAL_GATHER_BLOCKS=296" ""
  sweep "FRUGAL_GATHER_ROWS=4 FRUGAL_GATHER_BLOCKS=74" ""
  sweep FRUGAL_GATHER_ROWS=4 "--timer-every 8"
done
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "pipeline_modes or overlapped_pipeline_knobs" > gpurun_out/r2_c26_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c26_tests.log
