#!/bin/bash
# gather grid on the final source (environment knobs only), alternating, configs[1]
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null
O=gpurun_out/sweep_grid.txt; rm -f $O
run() { env $1 python bench.py --no-cpu-baseline --steps 300 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v})" >> $O; }
for i in 1 2; do
  run X=1
  run FRUGAL_GATHER_BLOCKS=148
  run FRUGAL_GATHER_BLOCKS=96
  run FRUGAL_GATHER_BLOCKS=192
  run FRUGAL_GATHER_BLOCKS=296
done
