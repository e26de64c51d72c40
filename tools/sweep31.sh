#!/bin/bash
# expand with 4 positions per row group in flight, configs[1]/[2], one B200 (compare with profiles/r1_bench*.json)
run() {
    local cfg=$1; shift
    env "$@" python bench.py --config "$cfg" --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $*', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
}
run criteo_kaggle X=1; run avazu X=1; run criteo_kaggle X=2
ncu --metrics gpu__time_duration.sum --clock-control none --launch-skip 600 -c 300 --csv --log-file gpurun_out/launches43.csv python bench.py --steps 40 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
