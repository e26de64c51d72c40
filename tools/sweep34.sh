#!/bin/bash
# gather grid 74 / 120 / 148, repeated, configs[1] and configs[2], one B200
run() {
    local cfg=$1; shift
    env "$@" python bench.py --config "$cfg" --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $*', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
}
for i in 1 2; do for g in 74 120 148; do run criteo_kaggle FRUGAL_GATHER_BLOCKS=$g; done; done
for g in 74 120; do run avazu FRUGAL_GATHER_BLOCKS=$g; done
