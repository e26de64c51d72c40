#!/bin/bash
# Round profiles of the bench workload (configs[1], one B200), written to gpurun_out/:
#  launches.csv   ncu launch list (gpu__time_duration.sum, --clock-control none) of a steady-state
#                 window of the bench command (after the warm-up launches)
#  <kernel>.ncu-rep  ncu --set full of one steady-state launch of each top kernel
# Numbers printed by bench.py under ncu are not bench values.
set -x
B="python bench.py --steps 40 --warmup 3 --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum --clock-control none --launch-skip 600 -c 600 --csv \
    --log-file gpurun_out/launches.csv $B > gpurun_out/prof_launch.log 2>&1
for k in k_gather_uniq k_segreduce k_flush_rows k_dot_model k_expand k_segred_combine k_schedule; do
    ncu --set full --import-source on --clock-control none -k regex:$k --launch-skip 30 -c 1 \
        -o gpurun_out/$k -f $B > gpurun_out/prof_$k.log 2>&1
done
# KG glue (FB15k-shaped bench)
BK="python bench.py --config fb15k --steps 40 --warmup 3 --no-cpu-baseline"
for k in k_transe_pos k_transe_pairs_tiled k_transe_grads_tiled; do
    ncu --set full --import-source on --clock-control none -k regex:$k --launch-skip 30 -c 1 \
        -o gpurun_out/$k -f $BK > gpurun_out/prof_$k.log 2>&1
done
