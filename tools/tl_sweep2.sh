#!/bin/bash
# NOTE: historical sweep (results in profiles/); some knobs it sets were removed after the measurement
# does the gather run at its isolated (ncu) speed when the host link is idle before it?
for v in TL_SLEEP=0.002 "TL_SLEEP=0.002 FRUGAL_EXPERIMENT_NO_DRAIN=1" "TL_SLEEP=0.02"; do
  echo "== $v"; env $v python tools/timeline.py 2>&1 | tail -11
done
