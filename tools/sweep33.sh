#!/bin/bash
# final-code grid check: gather and drain grids, configs[1], one B200
run() {
    local cfg=$1; shift
    env "$@" python bench.py --config "$cfg" --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $*', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
}
run criteo_kaggle X=default
run criteo_kaggle FRUGAL_GATHER_BLOCKS=100
run criteo_kaggle FRUGAL_GATHER_BLOCKS=120
run criteo_kaggle FRUGAL_SIDE_BLOCKS=24
run criteo_kaggle FRUGAL_SIDE_BLOCKS=16
run criteo_kaggle X=default
