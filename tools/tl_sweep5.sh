#!/bin/bash
# two-pass gather, steady state
for v in X=default FRUGAL_GATHER_BLOCKS=74 FRUGAL_GATHER_BLOCKS=296 "FRUGAL_SIDE_INLINE=1 FRUGAL_SIDE_BLOCKS=148"; do
  echo "== $v"; env $v TL_STEPS=120 python tools/timeline.py 2>&1 | tail -11 | awk '{printf "%s %s | ", $1, $4} END {print ""}'
done
