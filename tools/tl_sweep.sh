#!/bin/bash
# NOTE: historical sweep (results in profiles/); some knobs it sets were removed after the measurement
# timelines under pipeline variants: which concurrency slows the gather?
for v in X=default FRUGAL_INGEST_SERIAL=1 FRUGAL_EXPERIMENT_NO_DRAIN=1 "FRUGAL_INGEST_SERIAL=1 FRUGAL_SIDE_INLINE=1"; do
  echo "== $v"; env $v python tools/timeline.py 2>&1 | tail -11
done
