#!/bin/bash
# gather with R rows in flight per lane group: grid sweep, configs[1]
run() { env "$@" python bench.py --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()}, {k: round(v) for k,v in d['rows_per_step'].items() if 'gather' in k})"; }
run X=default
run FRUGAL_GATHER_BLOCKS=148
run FRUGAL_GATHER_BLOCKS=296
run FRUGAL_GATHER_BLOCKS=592
run FRUGAL_GATHER_BLOCKS=148 FRUGAL_POOL_STEPS=120
