#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
timeout 2400 python -m pytest tests/test_gpu_parity.py -m gpu -q -x --durations=5 -k "not freebase and not avazu and not 100_steps_recorded" > gpurun_out/r2_c24_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c24_tests.log
for i in 1 2; do for v in "X=1" "FRUGAL_PACK_THREADS=512" "FRUGAL_PACK_THREADS=1024" "FRUGAL_PACK_BLOCKS=16"; do
  env $v python bench.py --no-cpu-baseline --steps 300 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v}, {k: round(v, 3) for k, v in d['flushing_threads'].items()})" >> gpurun_out/r2_c24_sweep.txt 2>&1
done; done
