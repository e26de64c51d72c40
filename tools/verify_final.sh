#!/bin/bash
# Final-code check on one B200: smoke, GPU parity tests, headline bench line.
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > gpurun_out/smoke_final.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputests_final.log 2>&1
python bench.py > gpurun_out/r1_bench_final.json 2> gpurun_out/rb_final.err
