timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gputests30.log 2>&1
# NOTE: historical sweep (results in profiles/); some knobs it sets were removed after the measurement
run() {
    local cfg=$1; shift
    env "$@" python bench.py --config "$cfg" --no-cpu-baseline --steps 200 --warmup 20 2>/dev/null |
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $*', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
}
{ run criteo_kaggle X=default; run criteo_kaggle FRUGAL_EXPERIMENT_NO_DRAIN=1; run criteo_kaggle X=default; } > gpurun_out/sweep25.txt 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --launch-skip 600 -c 300 --csv --log-file gpurun_out/launches30.csv python bench.py --steps 40 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
