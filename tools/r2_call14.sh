#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
cat /sys/kernel/mm/transparent_hugepage/enabled /sys/kernel/mm/transparent_hugepage/shmem_enabled > gpurun_out/r2_c14_thp.txt 2>&1
for v in "X=1" "FRUGAL_FLUSH_THREADS=2" "FRUGAL_FLUSH_THREADS=6" "FRUGAL_GATE_STRICT=1"; do
  env $v python bench.py --no-cpu-baseline --steps 300 --warmup 20 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v}, d['flushing_threads'])" >> gpurun_out/r2_c14_sweep.txt 2>&1
done
