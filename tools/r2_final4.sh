#!/bin/bash
# Round-2 final source (762d586919fe), one B200: the whole GPU suite and the bench lines not yet
# re-run on it (KG, configs[4]-shaped, 2 ranks sharing the GPU)
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null
O=gpurun_out/r4; rm -rf $O; mkdir -p $O
timeout 2400 python -m pytest tests -m gpu -q --durations=40 > $O/r2_gpu_tests.log 2>&1
echo "pytest rc=$?" >> $O/r2_gpu_tests.log
python bench.py --config fb15k > $O/r2_bench_fb15k.json 2>> $O/rb.err
python bench.py --config freebase --steps 100 --warmup 10 > $O/r2_bench_freebase.json 2>> $O/rb.err
FRUGAL_BENCH_SAME_DEVICE=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --dist-backend gloo --steps 50 --warmup 5 --no-cpu-baseline > $O/r2_bench_n2_samedev.json 2>> $O/rb.err
for a in 0.9 1.0 1.1 1.2; do
  timeout 1200 python bench.py --config criteo_tb --alpha $a --steps 200 --warmup 20 > $O/r2_bench_criteo_tb_a$a.json 2>> $O/rb.err
done
