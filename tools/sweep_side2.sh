#!/bin/bash
# NOTE: historical sweep (results in profiles/); some knobs it sets were removed after the measurement
run() { env "$@" python bench.py --no-cpu-baseline --steps 150 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
for prio in high normal low; do for b in 16 32 64 148; do run FRUGAL_SIDE_PRIO=$prio FRUGAL_SIDE_BLOCKS=$b; done; done
run FRUGAL_SIDE_PRIO=high FRUGAL_SIDE_BLOCKS=32 FRUGAL_NO_EARLY=1
run FRUGAL_SIDE_PRIO=high FRUGAL_SIDE_BLOCKS=64 FRUGAL_NO_EARLY=1
