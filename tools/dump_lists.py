"""Diagnostic (world 1): run the Criteo-Kaggle step (world 1) for S steps and write, per step, the
exact host-table row lists the library touches, in pipeline order: urgent flush (a10),
gather host reads (a4), deferred drain + age-outs (a11) -> tools/lay/{urgent,reads,drain}.i32
(per step: count, then ids), for replay by tools/zc_probe7 (isolated link rate)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

OUT = os.path.join(os.path.dirname(os.path.abspath(__file__)), "lay")
os.makedirs(OUT, exist_ok=True)
for f in ("urgent", "reads", "drain"):
    p = os.path.join(OUT, f + ".i32")
    if os.path.exists(p):
        os.remove(p)
from paper_conf_asplos_xiezggl25_b200 import frugal as F
from paper_conf_asplos_xiezggl25_b200 import workload as W
from paper_conf_asplos_xiezggl25_b200.harness import make_context

cfg = W.config("criteo_kaggle", world=1)
S, L = int(os.environ.get("DUMP_STEPS", "100")), cfg.lookahead
st = W.gen_stream(cfg, S + L + 2)
fr = make_context(st, flags=F.F_RECORD)
dev = torch.device("cuda", 0)
ids = torch.from_numpy(st.ids).to(dev)
x = torch.from_numpy(np.ascontiguousarray(st.x[:, 0])).to(dev)
y = torch.from_numpy(np.ascontiguousarray(st.y[:, 0])).to(dev)
emb = torch.empty(cfg.batch * cfg.slots, cfg.dim, device=dev)
grad = torch.empty_like(emb)
loss = torch.zeros(S + L + 2, dtype=torch.float64, device=dev)


def app(name, a):
    with open(os.path.join(OUT, name + ".i32"), "ab") as f:
        np.array([len(a)], np.int32).tofile(f)
        np.asarray(a, np.int32).tofile(f)


# host-read rows of the gather (reading R7'): distinct rows of the step, not hot, whose
# latest update left the dirty pool's window (every touched row is updated at its step)
hot = np.zeros(cfg.n_rows, bool)
hot[st.hot] = True
last = np.full(cfg.n_rows, -10**9, np.int64)
P = cfg.age_out + 3
for t in range(L):
    fr.prefetch(t, ids[t], st.counts[t])
for s in range(S):
    sch = {}
    fr.step(s, ids[s + L], st.counts[s + L])
    sch = fr.get_schedule()
    app("urgent", sch["urgent"])
    app("drain", np.concatenate([sch["deferred"], sch["ageout"]]))
    u = np.unique(st.ids[s, 0])
    app("reads", u[~hot[u] & (last[u] < s - P + 2)])
    last[u] = s
    fr.lookup(s, emb)
    fr.dot_model(s, emb, x[s], y[s], grad, loss[s:s + 1])
    fr.backward_update(s, grad)
torch.cuda.synchronize()
print("dumped", S, "steps to", OUT)
