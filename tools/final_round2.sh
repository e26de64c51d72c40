#!/bin/bash
# Final-code evidence after the glue auto policy: smoke, GPU parity suite, bench lines, launch list.
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > gpurun_out/smoke_final.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputests_final.log 2>&1
python bench.py > gpurun_out/r1_bench.json 2> gpurun_out/fr2.err
python bench.py --no-cpu-baseline --config avazu > gpurun_out/r1_bench_avazu.json 2>> gpurun_out/fr2.err
python bench.py --no-cpu-baseline --config fb15k > gpurun_out/r1_bench_fb15k.json 2>> gpurun_out/fr2.err
B="python bench.py --steps 40 --warmup 3 --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum --clock-control none --launch-skip 600 -c 600 --csv \
    --log-file gpurun_out/launches.csv $B > gpurun_out/prof_launch.log 2>&1
