#!/bin/bash
# Final-code round evidence on one B200: smoke, GPU parity tests, bench lines, launch list,
# ncu --set full of the glue (fused lookup variant).
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > gpurun_out/smoke_final.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputests_final.log 2>&1
python bench.py > gpurun_out/r1_bench.json 2> gpurun_out/fr.err
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r1_bench_reference.json 2>> gpurun_out/fr.err
python bench.py --no-cpu-baseline --config avazu > gpurun_out/r1_bench_avazu.json 2>> gpurun_out/fr.err
B="python bench.py --steps 40 --warmup 3 --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum --clock-control none --launch-skip 600 -c 600 --csv \
    --log-file gpurun_out/launches.csv $B > gpurun_out/prof_launch.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_dot_model --launch-skip 30 -c 1 \
    -o gpurun_out/k_dot_model_fused -f $B > gpurun_out/prof_dm.log 2>&1
