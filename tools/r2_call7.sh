#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
python tools/host_profile.py > gpurun_out/r2_c7_host.txt 2>&1
FRUGAL_NO_COPY_WAIT=1 python tools/host_profile.py >> gpurun_out/r2_c7_host.txt 2>&1
