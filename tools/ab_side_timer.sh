#!/bin/bash
# A/B on one box: the current source vs the same source with the side stream's wait and pack
# under one phase timer again (as before session 2's split), alternating, configs[1]
cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null
rm -rf /tmp/varB && mkdir -p /tmp/varB && cp -r paper_conf_asplos_xiezggl25_b200 include bench.py oracle __graft_entry__.py MEASURED_PEAKS.json profiles /tmp/varB/ 2>/dev/null
python - <<'PY'
p='/tmp/varB/paper_conf_asplos_xiezggl25_b200/csrc/runtime.cu'
s=open(p).read()
new='''        if (s >= 2) {
            Timer tw(c, PH_SIDE, sd);
            launch_wait_word(c, c->dfl_ctl + CTL_APPLIED_ALL, (uint32_t)(s - 1), sd);
        }
        Timer tm(c, PH_SIDE, sd);
'''
old='''        Timer tm(c, PH_SIDE, sd);
        if (s >= 2) launch_wait_word(c, c->dfl_ctl + CTL_APPLIED_ALL, (uint32_t)(s - 1), sd);
'''
assert new in s
s=s.replace(new,old,1)
open(p,'w').write(s)
PY
(cd /tmp/varB && python -m paper_conf_asplos_xiezggl25_b200.build --force > /dev/null)
O=gpurun_out/ab_side_timer.txt
run() { (cd $1 && python bench.py --no-cpu-baseline --steps 300 --warmup 20 2>/dev/null) | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$2', round(d['value']/1e6,3), 'e2e', round(d['e2e']['value']/1e6,3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if v})" >> $O; }
for i in 1 2 3 4; do run . A_split; run /tmp/varB B_single; done
