#!/bin/bash
# Round-2 final code on one B200, part 2: the bench lines (profiles/r2_bench*.json), after the
# ncu captures of this source were summarised into profiles/ncu_traffic.json
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null
O=gpurun_out
python bench.py > $O/r2_bench.json 2> $O/r2_rb.err
python bench.py --impl reference --steps 3 --warmup 3 > $O/r2_bench_reference.json 2>> $O/r2_rb.err
python bench.py --config avazu > $O/r2_bench_avazu.json 2>> $O/r2_rb.err
python bench.py --config fb15k > $O/r2_bench_fb15k.json 2>> $O/r2_rb.err
python bench.py --no-cpu-baseline --alpha 0.99 > $O/r2_bench_a099.json 2>> $O/r2_rb.err
python bench.py --no-cpu-baseline --alpha 0 > $O/r2_bench_a0.json 2>> $O/r2_rb.err
python bench.py --no-cpu-baseline --mode write_through > $O/r2_bench_wt.json 2>> $O/r2_rb.err
python bench.py --no-cpu-baseline --cache-refresh 50 > $O/r2_bench_dyn.json 2>> $O/r2_rb.err
python bench.py --no-cpu-baseline --drain gpu > $O/r2_bench_gpudrain.json 2>> $O/r2_rb.err
python bench.py --config freebase --steps 100 --warmup 10 > $O/r2_bench_freebase.json 2>> $O/r2_rb.err
FRUGAL_BENCH_SAME_DEVICE=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --dist-backend gloo --steps 50 --warmup 5 --no-cpu-baseline > $O/r2_bench_n2_samedev.json 2>> $O/r2_rb.err
python bench.py --no-cpu-baseline --age-out 40 > $O/r2_bench_ageout40.json 2>> $O/r2_rb.err
timeout 1500 python bench.py --config criteo_tb --alpha 0.9 --steps 200 --warmup 20 > $O/r2_bench_criteo_tb_a0.9.json 2>> $O/r2_rb.err
timeout 1500 python bench.py --config criteo_tb --alpha 1.2 --steps 200 --warmup 20 > $O/r2_bench_criteo_tb_a1.2.json 2>> $O/r2_rb.err
for f in $O/r2_bench*.json; do echo "$f $(head -c 220 $f)"; done
# (compute-sanitizer was closed on the GPU pool by the time of the final runs: rc 86, nothing ran;
#  the round's sanitizer evidence is profiles/r2_compute_sanitizer.txt, earlier code of the round)
