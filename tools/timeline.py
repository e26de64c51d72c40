"""Print a per-step timeline of all library streams (FRUGAL_F_TIMERS) for the Criteo-Kaggle
bench workload: which phase runs when, on which stream, in the steady state."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_asplos_xiezggl25_b200 import frugal as F
from paper_conf_asplos_xiezggl25_b200 import workload as W
from paper_conf_asplos_xiezggl25_b200.harness import make_context

SLEEP = float(os.environ.get("TL_SLEEP", "0"))
cfg = W.config("criteo_kaggle", world=1, **({"opt": os.environ["TL_OPT"], "lr": 1.0} if os.environ.get("TL_OPT") else {}))
S, L = int(os.environ.get("TL_STEPS", "60")), cfg.lookahead
st = W.gen_stream(cfg, S + L + 2)
fr = make_context(st, flags=F.F_TIMERS)
dev = torch.device("cuda", 0)
ids = torch.from_numpy(st.ids).to(dev)
x = torch.from_numpy(np.ascontiguousarray(st.x[:, 0])).to(dev)
y = torch.from_numpy(np.ascontiguousarray(st.y[:, 0])).to(dev)
emb = torch.empty(cfg.batch * cfg.slots, cfg.dim, device=dev)
grad = torch.empty_like(emb)
loss = torch.zeros(S + L + 2, dtype=torch.float64, device=dev)
for t in range(L):
    fr.prefetch(t, ids[t], st.counts[t])
FUSED = os.environ.get("TL_FUSED", "1") == "1"
host_ms = []
for s in range(S):
    h0 = time.perf_counter()
    fr.step(s, ids[s + L], st.counts[s + L])
    if SLEEP:  # diagnostic: let the step's flushes settle before the gather
        torch.cuda.synchronize()
        time.sleep(SLEEP)
    fr.lookup(s, None if FUSED else emb)
    fr.dot_model(s, None if FUSED else emb, x[s], y[s], grad, loss[s:s + 1])
    fr.backward_update(s, grad)
    host_ms.append((time.perf_counter() - h0) * 1e3)
    if s == S - 6:
        torch.cuda.synchronize()
        fr.get_stats()
torch.cuda.synchronize()
print("host enqueue ms/step (steady state, last 30): %.3f" % (sum(host_ms[-30:]) / 30))
tl = fr.get_timeline()
t00 = tl[0][1]
for name, a, b in tl:
    print(f"{name:10s} {a - t00:9.3f} {b - t00:9.3f}  {b - a:7.3f} ms  " + " " * int((a - t00) * 40) + "#" * max(1, int((b - a) * 40)))
