#!/bin/bash
# side-drain grid (zero-copy D2H writes compete with the backward's HBM traffic), configs[1], one B200
run() { env "$@" python bench.py --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
for b in 32 16 8 4 2 32; do run FRUGAL_SIDE_BLOCKS=$b; done
