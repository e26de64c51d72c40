#!/bin/bash
# NOTE: historical sweep (results in profiles/); some knobs it sets were removed after the measurement
# ingest kernels after the scheduler (default) vs after the gather, configs[1]/[2], one B200
run() {
    local cfg=$1; shift
    env "$@" python bench.py --config "$cfg" --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
}
for i in 1 2; do run criteo_kaggle X=default; run criteo_kaggle FRUGAL_INGEST_AT=lookup; done
run avazu X=default; run avazu FRUGAL_INGEST_AT=lookup
