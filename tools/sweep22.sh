#!/bin/bash
# drain intensity split: deadline-(s+1) part (FRUGAL_SIDE_FIRST_BLOCKS) vs the rest (FRUGAL_SIDE_BLOCKS), configs[1], one B200
run() {
    local cfg=$1; shift
    env "$@" python bench.py --config "$cfg" --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
}
run criteo_kaggle X=default
run criteo_kaggle FRUGAL_SIDE_FIRST_BLOCKS=40 FRUGAL_SIDE_BLOCKS=16
run criteo_kaggle FRUGAL_SIDE_FIRST_BLOCKS=40 FRUGAL_SIDE_BLOCKS=12
run criteo_kaggle FRUGAL_SIDE_FIRST_BLOCKS=74 FRUGAL_SIDE_BLOCKS=16
run criteo_kaggle FRUGAL_SIDE_FIRST_BLOCKS=12 FRUGAL_SIDE_BLOCKS=20
run criteo_kaggle X=default
