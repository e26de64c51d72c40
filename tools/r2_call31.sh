#!/bin/bash
# session 2, call 7: is the gather / update bound by address translation of random accesses
# over big footprints?  (diagnostic masks fold the footprint; results are wrong by design)
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null
rm -rf gpurun_out/r2_c31_*; mkdir -p gpurun_out/r2_c31_ncu
O=gpurun_out/r2_c31_sweep.txt
sweep() {  # "env..." "bench args"
  env $1 python bench.py --no-cpu-baseline --steps 300 --warmup 20 $2 2>>gpurun_out/r2_c31_err.txt | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1 $2', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), 'frac', round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v})" >> $O 2>&1
}
for i in 1 2; do
  sweep X=1 ""
  sweep FRUGAL_DIAG_G_MASK=1048575 ""
  sweep FRUGAL_DIAG_G_MASK=8388607 ""
  sweep FRUGAL_DIAG_HOST_MASK=1048575 ""
  sweep FRUGAL_DIAG_HOST_MASK=4194303 ""
  sweep "FRUGAL_DIAG_HOST_MASK=1048575 FRUGAL_DIAG_G_MASK=1048575" ""
done
B="python bench.py --steps 40 --warmup 3 --no-cpu-baseline"
for k in k_update1 k_dot_rg k_gather_uniq; do
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:$k --launch-skip 30 -c 1 -o gpurun_out/r2_c31_ncu/$k -f $B > gpurun_out/r2_c31_ncu/$k.log 2>&1
  ncu -i gpurun_out/r2_c31_ncu/$k.ncu-rep --page source --csv --print-units base > gpurun_out/r2_c31_ncu/$k.source.csv 2>> gpurun_out/r2_c31_ncu/$k.log
  ncu -i gpurun_out/r2_c31_ncu/$k.ncu-rep --page raw --csv --print-units base > gpurun_out/r2_c31_ncu/$k.raw.csv 2>> gpurun_out/r2_c31_ncu/$k.log
  rm -f gpurun_out/r2_c31_ncu/$k.ncu-rep
done
