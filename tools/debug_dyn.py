"""Debug (N3): per step, compare the rows the GPU gathered with the oracle's synchronous
values before the step; report the first mismatching rows and their cache history."""
import sys
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from oracle.oracle import Oracle
from paper_conf_asplos_xiezggl25_b200 import workload as W
from paper_conf_asplos_xiezggl25_b200 import frugal as F
from paper_conf_asplos_xiezggl25_b200.harness import Trainer, make_context

cfg = W.config("tiny", world=1, lookahead=4, age_out=3, cache_ratio=0.05)
st = W.gen_stream(cfg, 60)
dyn = W.with_dynamic_hot(st, epoch=7)
fr = make_context(dyn, flags=F.F_RECORD)
o = Oracle(dyn)
tr = Trainer(fr, dyn)
epochs = [(0, set(dyn.hot.tolist()))] + [(t0, set(np.asarray(h).tolist())) for t0, h in dyn.hot_schedule]
hist = {}
for s in range(dyn.steps):
    ids = dyn.ids[s, 0]
    wo, _ = o.read_rows(ids)
    tr.step()
    o.step()
    sch = o.schedule()
    for k in sch["transition"].tolist():
        hist.setdefault(k, []).append(("X", s))
    for k in sch["urgent"].tolist():
        hist.setdefault(k, []).append(("U", s))
    for k, p in zip(sch["deferred"].tolist(), sch["deferred_p"].tolist()):
        hist.setdefault(k, []).append(("D", s, p))
    for k in sch["ageout"].tolist():
        hist.setdefault(k, []).append(("A", s))
    for k in set(ids.tolist()):
        hist.setdefault(k, []).append(("r", s))
    torch.cuda.synchronize()
    emb = tr.emb.cpu().numpy()
    bad = np.nonzero(np.abs(emb - wo).max(1) > 0)[0]
    if len(bad):
        ks = sorted(set(ids[bad].tolist()))
        print("step", s, "mismatching rows", ks[:10])
        for k in ks[:4]:
            print("  row", k, "hot by epoch:", [(t0, k in h) for t0, h in epochs if t0 <= s + 1],
                  "history:", hist.get(k, [])[-12:])
        break
else:
    print("no mismatch in", dyn.steps, "steps")
