#!/bin/bash
# one-launch chunk-task segment reduce + R-row gather
run() { env "$@" python bench.py --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()}, {k: round(v) for k,v in d['rows_per_step'].items() if 'gather' in k or 'long' in k})"; }
run X=default
run FRUGAL_GATHER_BLOCKS=148
run X=default
run FRUGAL_GATHER_BLOCKS=148
