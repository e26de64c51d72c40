#!/bin/bash
run() { env "$@" python bench.py --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
for gb in 32 74; do
run FRUGAL_GATHER_BLOCKS=$gb
run FRUGAL_GATHER_BLOCKS=$gb FRUGAL_EARLY=1
run FRUGAL_GATHER_BLOCKS=$gb FRUGAL_EARLY=1 FRUGAL_SIDE_BLOCKS=74
done
FRUGAL_EARLY=1 python tools/timeline.py > gpurun_out/timeline_early2.txt 2>&1
