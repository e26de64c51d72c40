#!/bin/bash
# NOTE: historical sweep (results in profiles/); some knobs it sets were removed after the measurement
# KG glue outputs per thread (FRUGAL_KG_TILE), FB15k / Freebase shapes, one B200
run() {
    local cfg=$1; shift
    env "$@" python bench.py --config "$cfg" --no-cpu-baseline --steps 100 --warmup 10 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $*', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), 'roofline', d['roofline']['bound'], round(d['roofline']['frac'] or 0, 3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
}
for t in 12 21; do FRUGAL_KG_TILE=$t timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "kg" 2>&1 | tail -1; done
for t in 22 12 21 22; do run fb15k FRUGAL_KG_TILE=$t; done
