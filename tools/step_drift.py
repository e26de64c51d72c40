"""Per-step phase durations over a long run (FRUGAL_F_TIMERS): does the step slow down as
training proceeds?  Every 10 steps: synchronize, read the timeline of those 10 steps,
print the mean gather / side / segred / step time and the host-table rows touched so far."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_asplos_xiezggl25_b200 import frugal as F
from paper_conf_asplos_xiezggl25_b200 import workload as W
from paper_conf_asplos_xiezggl25_b200.harness import make_context

cfg = W.config(os.environ.get("DRIFT_CONFIG", "criteo_kaggle"), world=1)
S, L = int(os.environ.get("DRIFT_STEPS", "300")), cfg.lookahead
CYCLE = int(os.environ.get("DRIFT_CYCLE", "0"))  # >0: reuse the first CYCLE batches (as bench.py)
G = CYCLE if CYCLE else S + L + 2
st = W.gen_stream(cfg, G)
fr = make_context(st, flags=F.F_TIMERS)
dev = torch.device("cuda", 0)
ids = torch.from_numpy(st.ids).to(dev)
x = torch.from_numpy(np.ascontiguousarray(st.x[:, 0])).to(dev)
y = torch.from_numpy(np.ascontiguousarray(st.y[:, 0])).to(dev)
emb = torch.empty(cfg.batch * cfg.slots, cfg.dim, device=dev)
grad = torch.empty_like(emb)
loss = torch.zeros(S + L + 2, dtype=torch.float64, device=dev)
for t in range(L):
    fr.prefetch(t, ids[t % G], st.counts[t % G])
seen = np.zeros(cfg.n_rows, bool)
torch.cuda.synchronize()
fr.get_timeline()
fr.get_stats()
prev = dict(fr.get_stats()["count"])
t_last = time.perf_counter()
for s in range(S):
    fr.step(s, ids[(s + L) % G], st.counts[(s + L) % G])
    fr.lookup(s, emb)
    fr.dot_model(s, emb, x[s % G], y[s % G], grad, loss[s:s + 1])
    fr.backward_update(s, grad)
    seen[st.ids[s % G].reshape(-1)] = True
    if (s + 1) % 10 == 0:
        torch.cuda.synchronize()
        now = time.perf_counter()
        tl = fr.get_timeline()
        stt = fr.get_stats()
        ph = {k: v / 10 for k, v in stt["ms"].items()}
        c = {k: v - prev.get(k, 0) for k, v in stt["count"].items()}
        prev = dict(stt["count"])
        print(f"steps {s - 8:4d}-{s + 1:4d}  wall/step {1e3 * (now - t_last) / 10:6.3f} ms  gather {ph['gather']:.3f}"
              f"  side {ph['side']:.3f}  segred {ph['segred']:.3f}  opt {ph['optimizer']:.3f}  ingest {ph['ingest']:.3f}"
              f"  host rows/step {c['gather_host'] / 10:8.0f}  side rows/step {(c['side_cold'] + c['side_hot']) / 10:8.0f}"
              f"  rows seen {seen.mean():.3f}", flush=True)
        t_last = time.perf_counter()
