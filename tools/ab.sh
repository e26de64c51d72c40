#!/bin/bash
# A/B: committed HEAD (ab_old/) vs working tree, same bench.py (hot-set window excluded)
run() { (cd $1 && python bench.py --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null) | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
for i in 1 2; do run ab_old; run .; done
