#!/bin/bash
# NOTE: historical sweep (results in profiles/); some knobs it sets were removed after the measurement
# split gather (HBM rows on a full grid + host rows on the zero-copy grid) vs one kernel, configs[1]/[2], one B200
run() {
    local cfg=$1; shift
    env "$@" python bench.py --config "$cfg" --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $*', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
}
for i in 1 2; do run criteo_kaggle FRUGAL_SPLIT_GATHER=1; run criteo_kaggle FRUGAL_SPLIT_GATHER=0; done
run criteo_kaggle FRUGAL_SPLIT_GATHER=1 FRUGAL_GATHER_BLOCKS=148
run avazu FRUGAL_SPLIT_GATHER=1; run avazu FRUGAL_SPLIT_GATHER=0
