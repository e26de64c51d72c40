"""Small world-1 run of the default path (flushing-thread drain, ingest graphs, fused lookup,
one-launch update) for compute-sanitizer: 30 steps of configs[0]'s table, then the final flush and a
check against the oracle.  `SAN_GPU_DRAIN=1` selects FRUGAL_F_GPU_DRAIN, `SAN_FUSED=0` the expand."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

from oracle.oracle import Oracle
from paper_conf_asplos_xiezggl25_b200 import frugal as F
from paper_conf_asplos_xiezggl25_b200 import workload as W
from paper_conf_asplos_xiezggl25_b200.harness import Trainer, make_context

cfg = W.config("tiny", world=1, batch=128, lookahead=4, age_out=2)
st = W.gen_stream(cfg, int(os.environ.get("SAN_STEPS", "30")))
flags = F.F_TIMERS | (F.F_GPU_DRAIN if os.environ.get("SAN_GPU_DRAIN") == "1" else 0)
fr = make_context(st, flags=flags)
tr = Trainer(fr, st, fused_lookup=os.environ.get("SAN_FUSED", "1") == "1", device_inputs=True)
tr.run()
fr.flush()
o = Oracle(st)
o.run()
ks = np.arange(cfg.n_rows)
w, _ = fr.read_host(ks)
wo, _ = o.read_rows(ks)
fr.close()
print("sanitize run: tables equal" if np.array_equal(w, wo) else f"sanitize run: MISMATCH {np.abs(w - wo).max()}")
