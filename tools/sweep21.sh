#!/bin/bash
# flushes by TMA bulk stores (FRUGAL_FLUSH_TMA: 0 none, 1 side drain, 2 all) x drain grid, configs[1]/[2], one B200
run() {
    local cfg=$1; shift
    env "$@" python bench.py --config "$cfg" --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
}
run criteo_kaggle FRUGAL_FLUSH_TMA=0
run criteo_kaggle FRUGAL_FLUSH_TMA=1
run criteo_kaggle FRUGAL_FLUSH_TMA=2
run criteo_kaggle FRUGAL_FLUSH_TMA=1 FRUGAL_SIDE_BLOCKS=32
run criteo_kaggle FRUGAL_FLUSH_TMA=1 FRUGAL_SIDE_BLOCKS=48
run criteo_kaggle FRUGAL_FLUSH_TMA=0
run criteo_kaggle FRUGAL_FLUSH_TMA=1
run avazu FRUGAL_FLUSH_TMA=0
run avazu FRUGAL_FLUSH_TMA=1
