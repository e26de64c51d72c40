#!/bin/bash
# Round profiles of one bench config on one B200 -> gpurun_out/prof_<config>/:
#  launches.csv       ncu launch list (gpu__time_duration.sum, --clock-control none) of a
#                     steady-state window of the bench command (after the warm-up launches)
#  <kernel>.csv       ncu --set full of 3 steady-state launches of each top kernel, exported
#                     in base units (--print-units base) for tools/ncu_summary.py
# Numbers printed by bench.py under ncu are not bench values.
#   tools/profile_round.sh [config] [extra bench flags]
CFG=${1:-criteo_kaggle}; shift
OUT=gpurun_out/prof_$CFG
mkdir -p $OUT
B="python bench.py --config $CFG --steps 40 --warmup 3 --no-cpu-baseline $*"
ncu --metrics gpu__time_duration.sum --clock-control none --launch-skip 600 -c 600 --csv \
    --log-file $OUT/launches.csv $B > $OUT/launch.log 2>&1
if [[ $CFG == fb15k || $CFG == freebase ]]; then
    KS="k_transe_pos k_transe_pairs_tiled k_transe_grads_tiled k_gather_uniq k_segreduce k_flush_rows"
else
    KS="k_gather_uniq k_update1 k_pack_drain k_dot_rg k_schedule k_radix_scatter k_dedup_emit k_flush_rows"
fi
for k in $KS; do
    ncu --set full --import-source on --clock-control none -k regex:$k --launch-skip 30 -c 3 \
        -o $OUT/$k -f $B > $OUT/$k.log 2>&1
    ncu -i $OUT/$k.ncu-rep --page raw --csv --print-units base > $OUT/$k.csv 2>> $OUT/$k.log
    ncu -i $OUT/$k.ncu-rep --page source --csv --print-units base > $OUT/$k.source.csv 2>> $OUT/$k.log
    rm -f $OUT/$k.ncu-rep  # gpurun copies back <= 64 MiB: keep the exported pages only
done
