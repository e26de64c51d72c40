#!/bin/bash
# side-drain grid around the sweet spot, configs[1] and configs[2], one B200
run() {
    local cfg=$1; shift
    env "$@" python bench.py --config "$cfg" --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
}
for b in 12 16 20 24 16; do run criteo_kaggle FRUGAL_SIDE_BLOCKS=$b; done
for b in 32 16 24; do run avazu FRUGAL_SIDE_BLOCKS=$b; done
