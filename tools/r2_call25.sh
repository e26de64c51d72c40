#!/bin/bash
# session 2, call 1: validate HEAD (smoke, quick parity), host-enqueue profile, pack-serial sweep
cd "${GRAFT_REPO_ROOT:-.}"
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2_c25_smoke.log 2>&1
python tools/host_profile.py > gpurun_out/r2_c25_host_profile.txt 2>&1
sweep() {  # label env...
  env "$@" python bench.py --no-cpu-baseline --steps 300 --warmup 20 2>>gpurun_out/r2_c25_err.txt | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), 'frac', round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v}, {k: round(v, 3) for k, v in d['flushing_threads'].items()})" >> gpurun_out/r2_c25_sweep.txt 2>&1
}
for i in 1 2; do
  sweep X=1
  sweep FRUGAL_PACK_SERIAL=1
  sweep FRUGAL_PACK_SERIAL=1 FRUGAL_PACK_BLOCKS=32
  sweep FRUGAL_PACK_SERIAL=1 FRUGAL_PACK_BLOCKS=148
  sweep FRUGAL_PACK_SERIAL=1 FRUGAL_PACK_BLOCKS=32 FRUGAL_PACK_ROWS=4
  sweep FRUGAL_PACK_SERIAL=1 FRUGAL_PACK_BLOCKS=148 FRUGAL_PACK_ROWS=4
  sweep FRUGAL_PACK_BLOCKS=8 FRUGAL_PACK_ROWS=4
done
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -x --durations=5 -k "not freebase and not avazu and not 100_steps" > gpurun_out/r2_c25_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c25_tests.log
