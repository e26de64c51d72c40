#!/bin/bash
# configs[4] (CriteoTB-shaped, d 128, SGD, cache 10 %) rows scaled to this host's memory; skew sweep
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
free -g > gpurun_out/r2_tb_free.txt
for a in 0.9 1.0 1.1 1.2; do
  timeout 1200 python bench.py --config criteo_tb --alpha $a --steps 200 --warmup 20 > gpurun_out/r2_bench_criteo_tb_a$a.json 2> gpurun_out/r2_bench_criteo_tb_a$a.err
done
