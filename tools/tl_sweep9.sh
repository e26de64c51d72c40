#!/bin/bash
# steady state, all serial: Adagrad (G in HBM, 4.3 GB randomly touched) vs SGD (no G)
S="FRUGAL_INGEST_SERIAL=1 FRUGAL_SIDE_INLINE=1 FRUGAL_SIDE_BLOCKS=148"
for v in "$S" "$S TL_OPT=sgd" "X=default" "TL_OPT=sgd"; do
  echo "== $v"; env $v TL_STEPS=120 python tools/timeline.py 2>&1 | tail -11 | awk '{printf "%s %s | ", $1, $4} END {print ""}'
done
