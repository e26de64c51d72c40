#!/bin/bash
# Round bench lines (one B200) -> gpurun_out/r1_bench*.json; then parity tests and smoke.
set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_final.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputests_final.log 2>&1
python bench.py > gpurun_out/r1_bench.json 2> gpurun_out/rb.err
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r1_bench_reference.json 2>> gpurun_out/rb.err
python bench.py --no-cpu-baseline --config avazu > gpurun_out/r1_bench_avazu.json 2>> gpurun_out/rb.err
python bench.py --no-cpu-baseline --mode write_through > gpurun_out/r1_bench_wt.json 2>> gpurun_out/rb.err
python bench.py --no-cpu-baseline --alpha 0.99 > gpurun_out/r1_bench_a099.json 2>> gpurun_out/rb.err
python bench.py --no-cpu-baseline --alpha 0 > gpurun_out/r1_bench_a0.json 2>> gpurun_out/rb.err
python bench.py --no-cpu-baseline --cache-refresh 50 > gpurun_out/r1_bench_dyn.json 2>> gpurun_out/rb.err
python bench.py --no-cpu-baseline --host-layout freq > gpurun_out/r1_bench_layout_freq.json 2>> gpurun_out/rb.err
python bench.py --no-cpu-baseline --config fb15k > gpurun_out/r1_bench_fb15k.json 2>> gpurun_out/rb.err
python bench.py --no-cpu-baseline --config freebase --steps 100 --warmup 10 > gpurun_out/r1_bench_freebase.json 2>> gpurun_out/rb.err
