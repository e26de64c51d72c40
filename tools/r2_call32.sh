#!/bin/bash
# session 2, call 8: k_update1 with dynamic work fetching (FRUGAL_UPDATE_DYN, default) vs static
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null
rm -rf gpurun_out/r2_c32_*; mkdir -p gpurun_out/r2_c32_ncu
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "pipeline_modes or overlapped_pipeline or criteo_kaggle_overlapped or tiny" > gpurun_out/r2_c32_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2_c32_tests.log
O=gpurun_out/r2_c32_sweep.txt
sweep() {  # "env..." "bench args"
  env $1 python bench.py --no-cpu-baseline --steps 300 --warmup 20 $2 2>>gpurun_out/r2_c32_err.txt | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1 $2', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), 'frac', round(d['roofline']['frac'],3), 'segred frac', round(d['rooflines']['segred']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v})" >> $O 2>&1
}
for i in 1 2 3; do
  sweep X=1 ""
  sweep FRUGAL_UPDATE_DYN=0 ""
done
sweep X=1 "--config avazu"
sweep FRUGAL_UPDATE_DYN=0 "--config avazu"
B="python bench.py --steps 40 --warmup 3 --no-cpu-baseline"
for v in 1 0; do
  FRUGAL_UPDATE_DYN=$v timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_update1 --launch-skip 30 -c 1 -o gpurun_out/r2_c32_ncu/upd$v -f $B > gpurun_out/r2_c32_ncu/upd$v.log 2>&1
  ncu -i gpurun_out/r2_c32_ncu/upd$v.ncu-rep --page source --csv --print-units base > gpurun_out/r2_c32_ncu/upd$v.source.csv 2>> gpurun_out/r2_c32_ncu/upd$v.log
  ncu -i gpurun_out/r2_c32_ncu/upd$v.ncu-rep --page raw --csv --print-units base > gpurun_out/r2_c32_ncu/upd$v.raw.csv 2>> gpurun_out/r2_c32_ncu/upd$v.log
  rm -f gpurun_out/r2_c32_ncu/upd$v.ncu-rep
done
