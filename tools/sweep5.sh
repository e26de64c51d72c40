#!/bin/bash
# NOTE: historical sweep (results in profiles/); some knobs it sets were removed after the measurement
run() { env "$@" python bench.py --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
for gb in 74 148 296; do for sb in 32 148; do
run FRUGAL_GATHER_BLOCKS=$gb FRUGAL_SIDE_BLOCKS=$sb
run FRUGAL_GATHER_BLOCKS=$gb FRUGAL_SIDE_BLOCKS=$sb FRUGAL_NO_EARLY=1
run FRUGAL_GATHER_BLOCKS=$gb FRUGAL_SIDE_BLOCKS=$sb FRUGAL_NO_EARLY=1 FRUGAL_DRAIN_AT=sched
done; done
