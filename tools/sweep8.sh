#!/bin/bash
run() { env "$@" python bench.py --no-cpu-baseline --steps 200 --warmup 20 2>gpurun_out/sweep8.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"; }
run X=base
for b in 32 74 148; do run FRUGAL_EARLY=1 FRUGAL_EARLY_BLOCKS=$b; done
run X=base
