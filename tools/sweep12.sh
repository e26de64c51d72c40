#!/bin/bash
# N3 dynamic cache vs static, configs[1], steady state
run() { python bench.py --no-cpu-baseline --steps 200 --warmup 20 "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['rows_per_step']; print('$*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v}, 'host', round(r['gather_host']), 'cache', round(r['gather_cache']), 'pool', round(r['gather_pool']), 'X', round(r['transition_hot']+r['transition_cold']), 'side', round(r['side_cold']+r['side_hot']))"; }
run
run --cache-refresh 50
run --cache-refresh 20
