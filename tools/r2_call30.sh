#!/bin/bash
# session 2, call 6: drain moved D2H by the copy engine (FRUGAL_PACK_CE), issued by a flushing thread
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null
rm -f gpurun_out/r2_c30_*
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "pipeline_modes or overlapped_pipeline" > gpurun_out/r2_c30_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c30_tests.log
O=gpurun_out/r2_c30_sweep.txt
sweep() {  # "env..." "bench args"
  env $1 python bench.py --no-cpu-baseline --steps 300 --warmup 20 $2 2>>gpurun_out/r2_c30_err.txt | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1 $2', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), 'frac', round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v}, {k: round(v, 3) for k, v in d['flushing_threads'].items()})" >> $O 2>&1
}
for i in 1 2; do
  sweep X=1 ""
  sweep FRUGAL_PACK_CE=1 ""
  sweep "FRUGAL_PACK_CE=1 FRUGAL_PACK_SERIAL=1" ""
  sweep "FRUGAL_PACK_CE=1 FRUGAL_FLUSH_THREADS=8" ""
  sweep "FRUGAL_PACK_CE=1 FRUGAL_EARLY=1 FRUGAL_EARLY_BLOCKS=64" ""
done
FRUGAL_PACK_CE=1 python tools/timeline.py > gpurun_out/r2_c30_timeline_ce.txt 2>&1
python tools/timeline.py > gpurun_out/r2_c30_timeline_default.txt 2>&1
