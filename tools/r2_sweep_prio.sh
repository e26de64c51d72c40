#!/bin/bash
# stream priorities on the final source (environment knobs only), alternating, configs[1]
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null
O=gpurun_out/sweep_prio.txt; rm -f $O
run() { env $1 python bench.py --no-cpu-baseline --steps 300 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v})" >> $O; }
for i in 1 2; do
  run X=1
  run FRUGAL_INGEST_PRIO=low
  run FRUGAL_INGEST_PRIO=high
  run FRUGAL_SIDE_PRIO=normal
  run "FRUGAL_INGEST_PRIO=low FRUGAL_SIDE_PRIO=low"
done
