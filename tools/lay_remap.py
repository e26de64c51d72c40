"""Diagnostic: map the exact host-row lists (tools/lay/*.i32, tools/dump_lists.py) through the
frequency-rank host layout (rank over the stream's first 50 steps, ties by id) -> *_freq.i32."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_xiezggl25_b200 import workload as W

D = os.path.join(os.path.dirname(os.path.abspath(__file__)), "lay")
cfg = W.config("criteo_kaggle", world=1)
ids = W.gen_ids(cfg, 50)
freq = np.bincount(ids.ravel(), minlength=cfg.n_rows)
order = np.argsort(-freq, kind="stable")
rank = np.empty(cfg.n_rows, np.int32)
rank[order] = np.arange(cfg.n_rows, dtype=np.int32)
for k in ("urgent", "reads", "drain"):
    a = np.fromfile(os.path.join(D, k + ".i32"), np.int32)
    out, i = [], 0
    while i < len(a):
        n = a[i]
        out.append(np.array([n], np.int32))
        out.append(np.sort(rank[a[i + 1:i + 1 + n]]))
        i += 1 + n
    np.concatenate(out).tofile(os.path.join(D, k + "_freq.i32"))
print("remapped")
