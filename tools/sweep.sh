#!/bin/bash
# Parameterised A/B sweep on one B200: every argument after the config is one variant, a
# space-separated list of environment assignments (knobs of DESIGN.md §10) and/or bench.py
# flags; each variant runs REPEAT times (alternating), one summary line per run.
#   tools/sweep.sh criteo_kaggle "X=default" "FRUGAL_SIDE_BLOCKS=32" "FRUGAL_GATHER_BLOCKS=148"
#   REPEAT=3 STEPS=300 tools/sweep.sh avazu "X=default" "--no-fused-lookup"
# (replaces the round-1 one-off scripts listed in tools/SWEEPS.md)
cfg=${1:?config}; shift
REPEAT=${REPEAT:-2}; STEPS=${STEPS:-200}; WARMUP=${WARMUP:-20}
for i in $(seq "$REPEAT"); do
  for v in "$@"; do
    envs=(); flags=(); prev=""
    for tok in $v; do  # --flag [value] go to bench.py, NAME=value to the environment
      if [[ $tok == --* ]]; then flags+=("$tok"); prev=flag
      elif [[ $tok == *=* ]]; then envs+=("$tok"); prev=""
      elif [[ $prev == flag ]]; then flags+=("$tok"); prev=""
      else envs+=("$tok"); fi
    done
    env "${envs[@]}" python bench.py --config "$cfg" --no-cpu-baseline --steps "$STEPS" --warmup "$WARMUP" \
        "${flags[@]}" 2>/dev/null |
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg', '$v', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v})"
  done
done
