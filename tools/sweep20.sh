#!/bin/bash
# host-table layout: id order vs frequency order (frugal_config.host_order), configs[1]/[2], one B200
run() {
    local cfg=$1; shift
    python bench.py --config "$cfg" --no-cpu-baseline --steps 200 --warmup 20 "$@" 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $*', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
}
for i in 1 2; do run criteo_kaggle --host-layout id; run criteo_kaggle --host-layout freq; done
run avazu --host-layout id; run avazu --host-layout freq
