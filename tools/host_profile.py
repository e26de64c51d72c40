"""Host-side cost of the per-step C-ABI calls on the bench workload (configs[1], world 1, fused
lookup, device-resident inputs): mean microseconds spent in each call, and the GPU time per step,
with and without FRUGAL_F_TIMERS.  If the host time per step reaches the GPU time per step the
GPU starves (the library lets the host run about one step ahead)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_asplos_xiezggl25_b200 import frugal as F
from paper_conf_asplos_xiezggl25_b200 import workload as W
from paper_conf_asplos_xiezggl25_b200.harness import make_context

cfg = W.config(os.environ.get("HP_CONFIG", "criteo_kaggle"), world=1)
S, L = int(os.environ.get("HP_STEPS", "200")), cfg.lookahead
SG = 64
st = W.gen_stream(cfg, SG)
dev = torch.device("cuda", 0)
ids = torch.from_numpy(st.ids).to(dev)
x = torch.from_numpy(np.ascontiguousarray(st.x[:, 0])).to(dev)
y = torch.from_numpy(np.ascontiguousarray(st.y[:, 0])).to(dev)
grad = torch.empty(cfg.batch * cfg.slots, cfg.dim, device=dev)
loss = torch.zeros(S + L + 2, dtype=torch.float64, device=dev)
ids_l = [ids[t] for t in range(SG)]                 # tensor views made once (no per-step indexing)
cnt_l = [np.ascontiguousarray(st.counts[t], dtype=np.int32) for t in range(SG)]
for flags, name in [(F.F_TIMERS, "F_TIMERS"), (0, "no timers")]:
    fr = make_context(st, flags=flags)
    for t in range(L):
        fr.prefetch(t, ids_l[t % SG], cnt_l[t % SG])
    acc = np.zeros(4)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    W0 = 20
    for s in range(S):
        if s == W0:
            torch.cuda.synchronize()
            fr.get_stats()  # resets the counters (host wait included)
            e0.record()
            acc[:] = 0
        t0 = time.perf_counter()
        fr.step(s, ids_l[(s + L) % SG], cnt_l[(s + L) % SG])
        t1 = time.perf_counter()
        fr.lookup(s, None)
        t2 = time.perf_counter()
        fr.dot_model(s, None, x[s % SG], y[s % SG], grad, loss[s:s + 1])
        t3 = time.perf_counter()
        fr.backward_update(s, grad)
        t4 = time.perf_counter()
        acc += [t1 - t0, t2 - t1, t3 - t2, t4 - t3]
    fr.join(None)
    e1.record()
    torch.cuda.synchronize()
    n = S - W0
    us = acc / n * 1e6
    wait_us = fr.get_stats()["host_wait_ms"] / n * 1e3
    print(f"{name:10s} host us/call: step {us[0]:6.1f} lookup {us[1]:6.1f} dot_model {us[2]:6.1f} "
          f"backward {us[3]:6.1f}  total {us.sum():6.1f} (of which blocked on the device {wait_us:6.1f}: "
          f"enqueue cost {us.sum() - wait_us:6.1f})   GPU ms/step {e0.elapsed_time(e1) / n:.4f}", flush=True)
    fr.close()
