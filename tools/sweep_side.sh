#!/bin/bash
# side-drain configuration sweep (experiment)
for b in 8 16 32 64 148 592; do
  FRUGAL_SIDE_BLOCKS=$b python bench.py --no-cpu-baseline --steps 150 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('blocks $b', round(d['value']/1e6,2), d['phases_ms_per_step'])"
done
FRUGAL_SIDE_INLINE=1 FRUGAL_SIDE_BLOCKS=592 python bench.py --no-cpu-baseline --steps 150 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('inline 592', round(d['value']/1e6,2), d['phases_ms_per_step'])"
