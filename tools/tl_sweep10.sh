#!/bin/bash
# flush kernel with R rows in flight: serial and default pipelines, steady state
S="FRUGAL_INGEST_SERIAL=1 FRUGAL_SIDE_INLINE=1 FRUGAL_SIDE_BLOCKS=148"
for v in "$S" "X=default" "FRUGAL_SIDE_BLOCKS=64" "FRUGAL_SIDE_BLOCKS=148"; do
  echo "== $v"; env $v TL_STEPS=120 python tools/timeline.py 2>&1 | tail -11 | awk '{printf "%s %s | ", $1, $4} END {print ""}'
done
