#!/bin/bash
# bench phases vs timeline phases over a longer run
run() { env "$@" python bench.py --no-cpu-baseline --steps $STEPS --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$* steps $STEPS', round(d['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
STEPS=40 run X=1
STEPS=200 run X=1
for n in 60 240; do echo "== timeline $n"; TL_STEPS=$n python tools/timeline.py 2>&1 | tail -11 | awk '{print $1, $4}' | tr '\n' ' '; echo; done
