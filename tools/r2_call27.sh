#!/bin/bash
# session 2, call 3: what slows the in-step gather (0.155 ms vs 0.088 alone)? timeline + diagnostics
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
python tools/timeline.py > gpurun_out/r2_c27_timeline.txt 2>&1
O=gpurun_out/r2_c27_sweep.txt
sweep() {  # "env..." "bench args"
  env $1 python bench.py --no-cpu-baseline --steps 300 --warmup 20 $2 2>>gpurun_out/r2_c27_err.txt | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1 $2', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), 'frac', round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v}, {k: round(v, 3) for k, v in d['flushing_threads'].items()})" >> $O 2>&1
}
for i in 1 2; do
  sweep X=1 ""
  sweep FRUGAL_DIAG_NO_APPLY=1 ""
  sweep "FRUGAL_DIAG_NO_APPLY=1 FRUGAL_PACK_SERIAL=1" ""
  sweep FRUGAL_INGEST_SERIAL=1 ""
  sweep FRUGAL_FLUSH_THREADS=1 ""
  sweep FRUGAL_FLUSH_THREADS=2 ""
  sweep FRUGAL_URGENT_SIDE=0 ""
done
FRUGAL_DIAG_NO_APPLY=1 FRUGAL_PACK_SERIAL=1 python tools/timeline.py > gpurun_out/r2_c27_timeline_noapply_serial.txt 2>&1
