#!/bin/bash
run() { env "$@" python bench.py --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
run X=base
for b in 8 16 32; do run FRUGAL_EARLY=1 FRUGAL_EARLY_BLOCKS=$b; done
run X=base
run FRUGAL_EARLY=1 FRUGAL_EARLY_BLOCKS=16 FRUGAL_DRAIN_AT=sched
FRUGAL_EARLY=1 FRUGAL_EARLY_BLOCKS=16 python tools/timeline.py > gpurun_out/timeline_early3.txt 2>&1
