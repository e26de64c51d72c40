#!/bin/bash
# NOTE: historical sweep (results in profiles/); some knobs it sets were removed after the measurement
run() { env "$@" python bench.py --no-cpu-baseline --steps 150 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
# (FRUGAL_EXPERIMENT_NO_DRAIN was removed; see profiles/r1_no_drain_upper_bound.txt)
# (FRUGAL_EXPERIMENT_NO_DRAIN was removed; see profiles/r1_no_drain_upper_bound.txt)
