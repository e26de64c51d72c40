#!/bin/bash
# gather grid with the current defaults (fused optimizer, 20-CTA drain), configs[1], one B200
run() {
    local cfg=$1; shift
    env "$@" python bench.py --config "$cfg" --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
}
for g in 74 148 296 74; do run criteo_kaggle FRUGAL_GATHER_BLOCKS=$g; done
