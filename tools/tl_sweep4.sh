#!/bin/bash
# steady-state (past the hot-set window) timelines: drain grid / placement
for v in X=default FRUGAL_SIDE_BLOCKS=148 "FRUGAL_SIDE_INLINE=1 FRUGAL_SIDE_BLOCKS=148" "FRUGAL_SIDE_INLINE=1 FRUGAL_SIDE_BLOCKS=148 FRUGAL_GATHER_BLOCKS=148" "FRUGAL_SIDE_INLINE=1 FRUGAL_SIDE_BLOCKS=296 FRUGAL_GATHER_BLOCKS=296"; do
  echo "== $v"; env $v TL_STEPS=120 python tools/timeline.py 2>&1 | tail -22 | awk '{printf "%s %s %s %s | ", $1, $2, $3, $4} END {print ""}'
done
