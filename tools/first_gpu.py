"""First GPU run: tiny world=1 stream, compare with the oracle (dev script)."""
import sys, time, traceback
import numpy as np, torch
sys.path.insert(0, ".")
from paper_conf_asplos_xiezggl25_b200 import workload as W, frugal as F
from paper_conf_asplos_xiezggl25_b200.harness import make_context, Trainer
from oracle.oracle import Oracle

def run(cfg, S, counts=None, flags=F.F_RECORD):
    st = W.gen_stream(cfg, S, counts=counts)
    o = Oracle(st)
    fr = make_context(st, flags=flags)
    tr = Trainer(fr, st)
    bad = 0
    for s in range(S):
        sched = {}
        tr.step(on_schedule=lambda s_: sched.update(fr.get_schedule()))
        o.step()
        osch = o.schedule()
        for key in ["urgent", "ageout"]:
            if sorted(sched[key].tolist()) != osch[key].tolist():
                bad += 1; print("MISMATCH", s, key, sorted(sched[key].tolist())[:10], osch[key].tolist()[:10])
        a = sorted(zip(sched["deferred"].tolist(), sched["deferred_p"].tolist()))
        b = sorted(zip(osch["deferred"].tolist(), osch["deferred_p"].tolist()))
        if a != b:
            bad += 1; print("MISMATCH deferred", s, a[:10], b[:10])
    fr.flush()
    ff = sorted(fr.get_final_flush().tolist()); off = o.final_flush().tolist()
    print("final flush equal:", ff == off, len(ff), len(off))
    ks = np.arange(cfg.n_rows)
    wg, Gg = fr.read_host(ks)
    wo, Go = o.read_rows(ks)
    print("max |w diff|", np.abs(wg - wo).max(), "max |G diff|", np.abs(Gg - Go).max(), "exact:", np.array_equal(wg, wo))
    lg = tr.losses(); lo = np.array([o.loss(s) for s in range(S)])
    print("loss max diff", np.abs(lg - lo).max(), lo[:3], lg[:3])
    print("sched mismatches", bad, "oracle violations", o.violations)
    fr.close()

try:
    c = W.config("tiny", world=1, lookahead=4, age_out=3)
    run(c, 30)
    c = W.config("tiny", world=1, lookahead=10, age_out=10, batch=64)
    rng = np.random.default_rng(0)
    run(c, 40, counts=rng.integers(0, 65, size=(40, 1)).astype(np.int32))
    c = W.config("criteo_kaggle", world=1)
    t = time.time(); st = W.gen_stream(c, 24); print("gen", time.time() - t)
    fr = make_context(st, flags=F.F_TIMERS)
    tr = Trainer(fr, st)
    tr.run(12); torch.cuda.synchronize(); fr.get_stats()
    t0 = time.time(); tr.run(24); torch.cuda.synchronize(); dt = time.time() - t0
    print("C2 n=1 wall per step ms", dt / 12 * 1e3, "samples/s", 12 * 8192 / dt)
    print(fr.get_stats())
except Exception:
    traceback.print_exc()
    sys.exit(1)
