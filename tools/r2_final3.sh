#!/bin/bash
# Round-2 final code (one side timer again), one B200: A/B of sampled phase timers, ncu captures of
# configs[1] / configs[2] summarised ON the box (so the bench lines that follow find their traffic),
# then the bench lines.  Copies profiles/ncu_traffic.json + summaries back through gpurun_out/.
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null
O=gpurun_out
rm -rf $O/prof_* $O/r3_*; mkdir -p $O/r3
run() { python bench.py --no-cpu-baseline --steps 300 --warmup 20 $2 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v})" >> $O/r3/ab_timer_every.txt; }
for i in 1 2 3; do run every1 ""; run every8 "--timer-every 8"; done
bash tools/profile_round.sh criteo_kaggle
bash tools/profile_round.sh avazu
for c in criteo_kaggle avazu; do
  python tools/ncu_summary.py $c profiles/r2_ncu_full_$c.txt $(ls $O/prof_$c/k_*.csv | grep -v source) > $O/r3/ns_$c.log 2>&1
  cp profiles/r2_ncu_full_$c.txt $O/r3/
  python tools/launch_summary.py $O/prof_$c/launches.csv > $O/r3/r2_launches_summary_$c.txt 2>&1
  cp $O/prof_$c/launches.csv $O/r3/r2_launches_$c.csv
done
cp profiles/ncu_traffic.json $O/r3/
python bench.py > $O/r3/r2_bench.json 2> $O/r3/rb.err
python bench.py --impl reference --steps 3 --warmup 3 > $O/r3/r2_bench_reference.json 2>> $O/r3/rb.err
python bench.py --config avazu > $O/r3/r2_bench_avazu.json 2>> $O/r3/rb.err
python bench.py --no-cpu-baseline --alpha 0.99 > $O/r3/r2_bench_a099.json 2>> $O/r3/rb.err
python bench.py --no-cpu-baseline --alpha 0 > $O/r3/r2_bench_a0.json 2>> $O/r3/rb.err
python bench.py --no-cpu-baseline --mode write_through > $O/r3/r2_bench_wt.json 2>> $O/r3/rb.err
python bench.py --no-cpu-baseline --cache-refresh 50 > $O/r3/r2_bench_dyn.json 2>> $O/r3/rb.err
python bench.py --no-cpu-baseline --drain gpu > $O/r3/r2_bench_gpudrain.json 2>> $O/r3/rb.err
python bench.py --no-cpu-baseline --age-out 40 > $O/r3/r2_bench_ageout40.json 2>> $O/r3/rb.err
python -c "import __graft_entry__ as g; g.smoke()" > $O/r3/r2_smoke.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tiny or overlapped or pipeline_modes" > $O/r3/r2_gpu_tests_quick.log 2>&1
echo "rc=$?" >> $O/r3/r2_gpu_tests_quick.log
