#!/bin/bash
# ncu --set full of one steady-state launch of each KG glue kernel (FB15k-shaped bench)
B="python bench.py --config fb15k --steps 40 --warmup 3 --no-cpu-baseline"
for k in k_transe_pos k_transe_pairs_tiled k_transe_grads_tiled; do
    ncu --set full --clock-control none -k regex:$k --launch-skip 30 -c 2 -o gpurun_out/$k -f $B > gpurun_out/prof_$k.log 2>&1
done
ncu --metrics gpu__time_duration.sum --clock-control none --launch-skip 600 -c 400 --csv --log-file gpurun_out/launches_kg.csv $B > /dev/null 2>&1
