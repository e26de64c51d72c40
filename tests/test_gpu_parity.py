"""Parity of the CUDA path (through the C ABI) against the CPU oracle, on a B200.

Bars (BASELINE.json north_star): dedup indices, priority-bucket membership, flush
sets bit-exact; fp32 tables (w, G) and per-step losses within 1e-5 max-abs after
100 steps.
"""
import dataclasses
import os

import numpy as np
import pytest

from oracle.oracle import Oracle
from paper_conf_asplos_xiezggl25_b200 import workload as W

pytestmark = pytest.mark.gpu
TOL = 1e-5


def _F():
    from paper_conf_asplos_xiezggl25_b200 import frugal as F
    return F


def run_parity(st, *, flags=None, mode=None, hot=None, check_dedup=True, check_sched=True, steps=None,
               sample_rows=None, oracle_kw=None, fused=False, on_step=None):
    """Run the stream on cuda:0 (world 1) and on the oracle; assert the bars."""
    F = _F()
    from paper_conf_asplos_xiezggl25_b200.harness import Trainer, make_context
    flags = F.F_RECORD if flags is None else flags
    mode = F.MODE_P2F if mode is None else mode
    hot = st.hot if hot is None else hot
    fr = make_context(st, flags=flags, mode=mode, hot=hot)
    o = Oracle(st, hot=hot, write_through=(mode == F.MODE_WRITE_THROUGH), **(oracle_kw or {}))
    tr = Trainer(fr, st, fused_lookup=fused)
    S = st.steps if steps is None else steps
    L = st.cfg.lookahead
    if check_dedup:
        for t in range(min(L, st.steps)):
            uq, inv = fr.get_dedup(t)
            ouq, oinv = o.dedup(t, 0)
            assert np.array_equal(uq, ouq) and np.array_equal(inv[:len(oinv)], oinv), f"dedup differs at {t}"
    gate_waits = 0
    for s in range(S):
        got = {}

        def cb(s_):
            if check_sched:
                got.update(fr.get_schedule())
                got["transition"] = fr.get_transition()
            if check_dedup and s_ + L < st.steps:
                t = s_ + L
                uq, inv = fr.get_dedup(t)
                ouq, oinv = o.dedup(t, 0)
                assert np.array_equal(uq, ouq), f"uniq differs at step {t}"
                assert np.array_equal(inv[:len(oinv)], oinv), f"inv differs at step {t}"

        tr.step(on_schedule=cb)
        o.step()
        if check_sched:
            ref = o.schedule()
            assert sorted(got["urgent"].tolist()) == ref["urgent"].tolist(), f"urgent set differs at {s}"
            assert sorted(zip(got["deferred"].tolist(), got["deferred_p"].tolist())) == \
                sorted(zip(ref["deferred"].tolist(), ref["deferred_p"].tolist())), f"deferred set differs at {s}"
            assert sorted(got["ageout"].tolist()) == ref["ageout"].tolist(), f"age-out set differs at {s}"
            assert sorted(got["transition"].tolist()) == ref["transition"].tolist(), f"transition differs at {s}"
            assert got["gate_wait"] == ref["gate_wait"]
            gate_waits += ref["gate_wait"]
            if on_step:
                on_step(s, got)
    assert o.violations == 0
    lo = np.array([o.loss(s) for s in range(S)])
    lg = tr.losses()[:S]
    assert np.abs(lg - lo).max() <= TOL, f"loss differs by {np.abs(lg - lo).max()}"
    out = dict(fr=fr, o=o, gate_waits=gate_waits)
    if S == st.steps:
        fr.flush()
        ff = o.final_flush()
        assert sorted(fr.get_final_flush().tolist()) == ff.tolist(), "final flush set differs"
        ks = np.arange(st.cfg.n_rows) if sample_rows is None else sample_rows
        w, G = fr.read_host(ks)
        wo, Go = o.read_rows(ks)
        out.update(dw=float(np.abs(w - wo).max()), dG=float(np.abs(G - Go).max()),
                   exact=bool(np.array_equal(w, wo) and np.array_equal(G, Go)), w=w, wo=wo)
        assert out["dw"] <= TOL and out["dG"] <= TOL, (out["dw"], out["dG"])
    else:
        ks = sample_rows
        w, G = fr.read_rows(ks)
        wo, Go = o.read_rows(ks)
        out.update(dw=float(np.abs(w - wo).max()), dG=float(np.abs(G - Go).max()))
        assert out["dw"] <= TOL and out["dG"] <= TOL, (out["dw"], out["dG"])
    return out


def run_overlapped(st, *, fused=True, flags=None, sample_rows=None, hot=None, exact=None, host_inputs=False):
    """The bench's launch configuration: FRUGAL_F_TIMERS only (no F_RECORD, so no
    per-step synchronisation), no per-step callbacks, ids / x / y resident in HBM and passed
    as device pointers -- the ingest of s+L, the side drain and the main stream overlap as in
    bench.py.  After frugal_flush: per-step losses, the final-flush set and the host table
    (w, G; all rows or `sample_rows`) against the oracle run to the end."""
    F = _F()
    from paper_conf_asplos_xiezggl25_b200.harness import Trainer, make_context
    flags = F.F_TIMERS if flags is None else flags
    hot = st.hot if hot is None else hot
    fr = make_context(st, flags=flags, hot=hot)
    tr = Trainer(fr, st, fused_lookup=fused, device_inputs=not host_inputs, host_inputs=host_inputs)
    tr.run()
    fr.flush()
    lg = tr.losses()
    o = Oracle(st, hot=hot)
    o.run()
    assert o.violations == 0
    lo = np.array([o.loss(s) for s in range(st.steps)])
    assert np.abs(lg - lo).max() <= TOL, f"loss differs by {np.abs(lg - lo).max()}"
    assert sorted(fr.get_final_flush().tolist()) == o.final_flush().tolist(), "final flush set differs"
    ks = np.arange(st.cfg.n_rows) if sample_rows is None else sample_rows
    w, G = fr.read_host(ks)
    wo, Go = o.read_rows(ks)
    dw, dG = float(np.abs(w - wo).max()), float(np.abs(G - Go).max())
    assert dw <= TOL and dG <= TOL, (dw, dG)
    if exact:
        assert np.array_equal(w, wo) and np.array_equal(G, Go), "tables are expected bit-exact"
    stats = fr.get_stats()
    fr.close()
    return dict(stats=stats, w=w, wo=wo)


def _touched_sample(st, steps, size, seed):
    rng = np.random.default_rng(seed)
    touched = np.unique(st.ids[:steps, 0].ravel())
    return np.sort(rng.choice(touched, size=min(size, len(touched)), replace=False))


def tiny1(**over):
    kw = dict(world=1)
    kw.update(over)
    return W.config("tiny", **kw)


def test_tiny_100_steps_parity():
    """configs[0] (tiny DLRM-style, 10^4 x 16, batch 256) at world 1, 100 parity steps."""
    st = W.gen_stream(tiny1(), 100)
    r = run_parity(st)
    w0 = np.array([[r["o"].init_value(k, j) for j in range(16)] for k in range(st.cfg.n_rows)], np.float32)
    assert np.abs(r["wo"] - w0).max() >= 1e-3  # non-vacuous: parameters moved
    assert r["gate_waits"] > 0                 # the gate actually blocked on urgent flushes
    assert r["exact"], "tables are expected bit-exact (canonical fixed-order arithmetic)"
    r["fr"].close()


def test_ragged_and_empty_batches():
    cfg = tiny1(batch=64, lookahead=5, age_out=2)
    rng = np.random.default_rng(7)
    counts = rng.integers(0, 65, size=(40, 1)).astype(np.int32)
    counts[3] = 0
    counts[10:12] = 0
    counts[-1] = 0
    counts[20] = 64
    st = W.gen_stream(cfg, 40, counts=counts)
    run_parity(st)["fr"].close()


@pytest.mark.parametrize("L,D", [(2, 1), (3, 5), (31, 1), (10, 40)])
def test_lookahead_and_ageout(L, D):
    st = W.gen_stream(tiny1(lookahead=L, age_out=D, batch=128), 50)
    run_parity(st)["fr"].close()


@pytest.mark.parametrize("dim", [4, 8, 64, 128, 400])
def test_dims(dim):
    cfg = W.WorkloadConfig("d", [3000, 500, 7], dim=dim, batch=96, world=1, lookahead=4, age_out=3)
    st = W.gen_stream(cfg, 25)
    run_parity(st)["fr"].close()


def test_sgd():
    st = W.gen_stream(tiny1(opt="sgd", lr=1.0, batch=128), 40)
    run_parity(st)["fr"].close()


def test_long_segments_chunked_order():
    """A 1-row and a 3-row table: segments of 1000+ occurrences exercise the chunked
    fixed-order reduction (R23) against the oracle bit for bit."""
    cfg = W.WorkloadConfig("long", [1, 3, 5000], dim=32, batch=1500, world=1, lookahead=3, age_out=2)
    st = W.gen_stream(cfg, 12)
    r = run_parity(st)
    assert r["exact"]
    r["fr"].close()


def test_metamorphic_tables_identical():
    """P2F == write-through (Frugal-Sync) == no cache == large cache == L=2, bit for bit."""
    F = _F()
    base = W.gen_stream(tiny1(batch=128, lookahead=6, age_out=3), 30)
    tabs = []
    variants = [dict(), dict(mode=F.MODE_WRITE_THROUGH), dict(hot=np.zeros(0, np.int64)),
                dict(hot=np.arange(0, 10_000, 2, dtype=np.int64))]
    for v in variants:
        r = run_parity(base, **v)
        tabs.append(r["w"])
        r["fr"].close()
    st2 = dataclasses.replace(base, cfg=dataclasses.replace(base.cfg, lookahead=2))
    r = run_parity(st2)
    tabs.append(r["w"])
    r["fr"].close()
    for t in tabs[1:]:
        assert np.array_equal(tabs[0], t)


def test_write_through_flushes_every_update():
    F = _F()
    st = W.gen_stream(tiny1(batch=64, lookahead=4), 10)
    r = run_parity(st, mode=F.MODE_WRITE_THROUGH)
    r["fr"].close()


def test_fused_lookup_parity():
    """Fused lookup (lookup/dot_model with NULL emb: the glue reads the gathered distinct
    rows through inv, no expand): tables, losses and sets bit-exact as with the expand."""
    st = W.gen_stream(tiny1(), 60)
    r = run_parity(st, fused=True)
    assert r["exact"]
    r["fr"].close()


@pytest.mark.parametrize("dim,tables", [(8, 3), (64, 5), (32, 40), (400, 3)])
def test_fused_lookup_shapes(dim, tables):
    """Every glue variant (J = 1..13 lanes per row, F <= 32 register-cached or F > 32)
    and ragged / empty batches with the fused lookup."""
    cfg = W.WorkloadConfig("fz", [500 + 37 * i for i in range(tables)], dim=dim, batch=64, world=1,
                           lookahead=4, age_out=3)
    rng = np.random.default_rng(dim + tables)
    counts = rng.integers(0, 65, size=(20, 1)).astype(np.int32)
    counts[5] = 0
    st = W.gen_stream(cfg, 20, counts=counts)
    run_parity(st, fused=True)["fr"].close()


def test_fused_lookup_errors():
    """dot_model's emb must be NULL exactly when lookup's out was."""
    F = _F()
    import torch
    from paper_conf_asplos_xiezggl25_b200.harness import make_context
    st = W.gen_stream(tiny1(batch=32, lookahead=3), 6)
    fr = make_context(st)
    for t in range(3):
        fr.prefetch(t, st.ids[t], st.counts[t])
    fr.step(0, st.ids[3], st.counts[3])
    fr.lookup(0, None)
    B, d = 32, st.cfg.dim
    emb = torch.empty(B * st.cfg.slots, d, device="cuda")
    x = torch.from_numpy(st.x[0, 0]).cuda()
    y = torch.from_numpy(st.y[0, 0]).cuda()
    loss = torch.zeros(1, dtype=torch.float64, device="cuda")
    with pytest.raises(F.FrugalError) as e:
        fr.dot_model(0, emb, x, y, emb, loss)
    assert e.value.status == -1
    with pytest.raises(F.FrugalError):
        fr.transe_model(0, None, 4, 1.0, emb, loss)
    fr.dot_model(0, None, x, y, emb, loss)
    fr.close()


def test_invalid_id_fails_loudly():
    F = _F()
    from paper_conf_asplos_xiezggl25_b200.harness import Trainer, make_context
    st = W.gen_stream(tiny1(batch=32, lookahead=3), 6)
    st.ids[4, 0, 5] = st.cfg.n_rows + 7
    fr = make_context(st)
    tr = Trainer(fr, st)
    with pytest.raises(F.FrugalError) as e:
        for _ in range(6):
            tr.step()
        fr.flush()
    assert e.value.status == -1
    fr.close()


def test_call_order_enforced():
    F = _F()
    import torch
    from paper_conf_asplos_xiezggl25_b200.harness import make_context
    st = W.gen_stream(tiny1(batch=32, lookahead=3), 6)
    fr = make_context(st)
    out = torch.empty(32, 16, device="cuda")
    with pytest.raises(F.FrugalError) as e:
        fr.lookup(0, out)
    assert e.value.status == -4
    with pytest.raises(F.FrugalError):
        fr.step(0, st.ids[3], st.counts[3])  # steps 0..L-1 not prefetched yet
    fr.close()


@pytest.mark.parametrize("kind", ["freq", "random_partial", "random_full"])
def test_host_layout_parity(kind):
    """frugal_config.host_order only moves bytes in the host table: every
    artefact, and the host table read back through the layout, match the oracle (which has
    no layout) exactly."""
    cfg = tiny1(batch=128, lookahead=4, age_out=2)
    st = W.gen_stream(cfg, 40)
    N = cfg.n_rows
    rng = np.random.default_rng(17)
    order = {"freq": lambda: W.host_order(cfg, st.ids[:10], st.counts[:10]),
             "random_partial": lambda: rng.permutation(N)[: N // 3],
             "random_full": lambda: rng.permutation(N)}[kind]().astype(np.int64)
    r = run_parity(dataclasses.replace(st, host_order=order))
    assert r["exact"]
    r["fr"].close()


def test_host_layout_errors():
    F = _F()
    from paper_conf_asplos_xiezggl25_b200.harness import make_context
    st = W.gen_stream(tiny1(batch=32, lookahead=3), 6)
    for bad in (np.array([3, 5, 3], np.int64), np.array([0, st.cfg.n_rows], np.int64)):
        with pytest.raises(F.FrugalError) as e:
            make_context(dataclasses.replace(st, host_order=bad))
        assert e.value.status == -1


@pytest.mark.parametrize("env", [{"FRUGAL_EARLY": "1", "FRUGAL_HOST_FLUSH": "0"}, {"FRUGAL_DRAIN_AT": "sched"},
                                 {"FRUGAL_EARLY": "1", "FRUGAL_DRAIN_AT": "sched", "FRUGAL_HOST_FLUSH": "0"},
                                 {"FRUGAL_SIDE_INLINE": "1"}, {"FRUGAL_SIDE_INLINE": "1", "FRUGAL_HOST_FLUSH": "0"},
                                 {"FRUGAL_NO_POOL_HITS": "1"}, {"FRUGAL_FUSE_OPT": "0"}, {"FRUGAL_UPDATE1": "0"},
                                 {"FRUGAL_FLUSH_TMA": "2", "FRUGAL_HOST_FLUSH": "0"},
                                 {"FRUGAL_EARLY": "1", "FUSED": "1", "FRUGAL_HOST_FLUSH": "0"},
                                 {"FRUGAL_GLUE_CACHE": "0", "FUSED": "1"}, {"FRUGAL_GLUE_CACHE": "1", "FUSED": "1"},
                                 {"FRUGAL_GLUE_CACHE": "0"}, {"FRUGAL_GLUE_RG": "0", "FUSED": "1"},
                                 {"FRUGAL_PACK_TMA": "1", "FUSED": "1"}, {"FRUGAL_PACK_2STAGE": "1", "FUSED": "1"},
                                 {"FRUGAL_PACK_ROWS": "4"}, {"FRUGAL_GRAPHS": "0"}, {"FRUGAL_URGENT_SIDE": "0"},
                                 {"FRUGAL_GATE_STRICT": "1"}, {"FRUGAL_GATHER_ROWS": "4", "FUSED": "1"},
                                 {"FRUGAL_GATHER_ROWS": "2"}, {"FRUGAL_PACK_SERIAL": "1", "FUSED": "1"},
                                 {"FRUGAL_GATHER_ROWS": "1", "FRUGAL_PACK_SERIAL": "0"},
                                 {"FRUGAL_EARLY": "1", "FUSED": "1"}, {"FRUGAL_EARLY": "1", "FRUGAL_EARLY_ROWS": "1"},
                                 {"FRUGAL_GLUE_UNROLL": "1", "FUSED": "1"}, {"FRUGAL_GLUE_UNROLL": "4"},
                                 {"FRUGAL_UPDATE_SHORT": "1", "FUSED": "1"}, {"FRUGAL_PACK_CE": "1"},
                                 {"FRUGAL_PACK_CE": "1", "FUSED": "1", "FRUGAL_FLUSH_THREADS": "3"},
                                 {"FRUGAL_UPDATE_DYN": "1", "FUSED": "1"}])
def test_pipeline_modes_parity(env):
    """The optional schedules (early gather of the next step, drain after the gather,
    inline drain) keep every artefact bit-exact (run in a subprocess: the knobs are read
    at context creation)."""
    import subprocess
    import sys
    code = ("import sys; sys.path.insert(0, '.');"
            "from tests.test_gpu_parity import run_parity, tiny1; from paper_conf_asplos_xiezggl25_b200 import workload as W;"
            "import os; st = W.gen_stream(tiny1(batch=128, lookahead=4, age_out=2), 40);"
            "r = run_parity(st, fused=bool(os.environ.get('FUSED'))); r['fr'].close();"
            "print('OK', r['exact'])")
    e = dict(os.environ)
    e.update(env)
    out = subprocess.run([sys.executable, "-c", code], env=e, capture_output=True, text=True,
                         cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))), timeout=600)
    assert "OK True" in out.stdout, out.stdout + out.stderr


@pytest.mark.parametrize("opt", ["adagrad", "sgd"])
def test_kg_transe_parity(opt):
    """KG workload (configs[3] shape, small): TransE glue with chunked shared negatives;
    entities and relations in one id space, slots (h, r, t, neg) -> tables (E, R, E, E)."""
    cfg = W.config("tiny_kg", opt=opt, lr=0.05 if opt == "adagrad" else 0.5)
    rng = np.random.default_rng(5)
    counts = rng.integers(0, cfg.batch + 1, size=(30, 1)).astype(np.int32)
    counts[4] = 0
    st = W.gen_stream(cfg, 30, counts=counts)
    r = run_parity(st)
    assert r["exact"]
    r["fr"].close()


def test_kg_transe_tiles_ragged():
    """Tiled TransE glue across tile boundaries: d = 72 (k tiles 32+32+8), chunks of 50 (b/j
    tiles 32+18) and a ragged last chunk of 30, bit-exact against the oracle."""
    cfg = W.config("tiny_kg", dim=72, neg_chunk=50, batch=130, table_rows=[3000, 30])
    st = W.gen_stream(cfg, 10)
    r = run_parity(st)
    assert r["exact"]
    r["fr"].close()



def test_fb15k_kg_full_size():
    """FB15k-shaped KG at full size (14,951 entities + 1,345 relations, d=400, batch 1200,
    chunks of 200 negatives): every artefact and the whole table against the oracle."""
    cfg = W.config("fb15k", world=1)
    st = W.gen_stream(cfg, 12)
    r = run_parity(st)
    assert r["exact"]
    r["fr"].close()


# ----------------------------------------------------------------------------- N3 dynamic cache
def test_dynamic_cache_parity():
    """SURVEY §8(f) N3 (reading R27): the hot set is recomputed every E steps from the
    previous window (LFU over a sliding window); every schedule artefact, the transition
    sets X(t0), the losses and the final tables match the oracle; the tables are also
    bit-identical to a static-cache run (values cannot depend on the cache)."""
    cfg = tiny1(lookahead=4, age_out=3, cache_ratio=0.05)
    st = W.gen_stream(cfg, 60)
    dyn = W.with_dynamic_hot(st, epoch=7)
    r = run_parity(dyn)
    assert r["exact"]
    c = r["fr"].get_stats()["count"]
    assert c["transition_hot"] + c["transition_cold"] > 0  # rows actually moved dirty
    r["fr"].close()
    s0 = run_parity(st, check_dedup=False)
    assert np.array_equal(s0["w"], r["w"])
    s0["fr"].close()


@pytest.mark.parametrize("seed", range(3))
def test_dynamic_cache_random_sets(seed):
    """Random hot sets (any turnover, growing and shrinking) at random epoch lengths > L."""
    rng = np.random.default_rng(900 + seed)
    L = int(rng.choice([2, 3, 5]))
    D = int(rng.choice([1, L, 2 * L]))
    cfg = tiny1(batch=48, lookahead=L, age_out=D, cache_ratio=0.05, seed_ids=seed + 11)
    st = W.gen_stream(cfg, 40)
    E = int(rng.integers(L + 1, L + 5))
    sched = []
    for t0 in range(E, st.steps, E):
        k = int(rng.integers(100, 600))  # <= the 625 slots (500 + 25%)
        sched.append((t0, np.sort(rng.choice(cfg.n_rows, size=k, replace=False)).astype(np.int64)))
    r = run_parity(dataclasses.replace(st, hot_schedule=sched))
    assert r["exact"]
    r["fr"].close()


def test_dynamic_cache_capacity_and_order_errors():
    F = _F()
    from paper_conf_asplos_xiezggl25_b200.harness import Trainer, make_context
    cfg = tiny1(lookahead=3)
    st = W.gen_stream(cfg, 10)
    fr = make_context(st)  # static cache: set_hot is refused
    with pytest.raises(F.FrugalError):
        fr.set_hot(5, st.hot)
    fr.close()
    fr = make_context(st, flags=F.F_DYNAMIC_CACHE)
    fr.set_hot(5, st.hot)
    with pytest.raises(F.FrugalError):  # one change already pending
        fr.set_hot(9, st.hot)
    fr.close()
    # far more rows than slots: detected on the device, reported by a following call
    big = dataclasses.replace(st, hot_schedule=[(5, np.arange(cfg.n_rows))])
    fr = make_context(big)
    tr = Trainer(fr, big)
    with pytest.raises(F.FrugalError, match="slots"):
        tr.run()
    fr.close()


# ----------------------------------------------------------------------------- overlapped pipeline
@pytest.mark.parametrize("fused", [False, True])
def test_overlapped_pipeline_tiny_100_steps(fused):
    """the exact-parity runs above record the schedule (F_RECORD synchronises
    after every scheduler), so they never overlap the ingest of s+L with the gather and the
    backward of s.  Here: the bench's configuration (F_TIMERS only, device-resident inputs,
    no callbacks), world 1, 100 steps; tables bit-exact."""
    st = W.gen_stream(tiny1(), 100)
    run_overlapped(st, fused=fused, exact=True)


@pytest.mark.parametrize("env", [{"FRUGAL_EARLY": "1"}, {"FRUGAL_DRAIN_AT": "sched"}, {"FRUGAL_FUSE_OPT": "0"},
                                 {"FRUGAL_GATHER_ROWS": "1", "FRUGAL_PACK_SERIAL": "0"},
                                 {"FRUGAL_GATHER_ROWS": "4", "FRUGAL_PACK_SERIAL": "1"},
                                 {"FRUGAL_EARLY": "1", "FRUGAL_EARLY_BLOCKS": "64"}, {"FRUGAL_GLUE_UNROLL": "1"},
                                 {"FRUGAL_UPDATE_SHORT": "1"}, {"FRUGAL_PACK_CE": "1"}, {"FRUGAL_UPDATE_DYN": "1"}])
def test_overlapped_pipeline_knobs(env):
    """The optional schedules of DESIGN.md §10 in the overlapped configuration (subprocess:
    the knobs are read at context creation)."""
    import subprocess
    import sys
    code = ("import sys; sys.path.insert(0, '.');"
            "from tests.test_gpu_parity import run_overlapped, tiny1; from paper_conf_asplos_xiezggl25_b200 import workload as W;"
            "st = W.gen_stream(tiny1(batch=128, lookahead=4, age_out=2), 60);"
            "run_overlapped(st, fused=True, exact=True); print('OK')")
    e = dict(os.environ)
    e.update(env)
    out = subprocess.run([sys.executable, "-c", code], env=e, capture_output=True, text=True,
                         cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))), timeout=600)
    assert "OK" in out.stdout, out.stdout + out.stderr


# ----------------------------------------------------------------------------- full size, 100 steps
def test_criteo_kaggle_100_steps_recorded():
    """configs[1] at full size (26 tables, 33.8M rows, d 32, batch 8192, cache 5 %, L 10,
    D 10), 100 steps (the north_star bar): dedup, every schedule set and the gate bit-exact
    at every step; losses within 1e-5; final-flush set exact; 20k sampled touched rows of
    the host table (w, G) within 1e-5 after the final flush.  Past step 11 rows are aged
    out, and 100 steps wrap each of the P = D+3 = 13 dirty-pool segments 7 times."""
    cfg = W.config("criteo_kaggle", world=1)
    st = W.gen_stream(cfg, 100)
    sample = _touched_sample(st, 100, 20000, 0)
    ages = []

    F = _F()
    r = run_parity(st, sample_rows=sample, fused=True, flags=F.F_RECORD,
                   on_step=lambda s, got: ages.append(len(got["ageout"])))
    c = r["fr"].get_stats()["count"]
    assert sum(ages[:cfg.age_out + 1]) == 0 and sum(ages) > 0, "age-out never exercised"
    assert c["gather_pool"] > 0 and st.steps > cfg.age_out + 3 + 1, "dirty pool never wrapped"
    r["fr"].close()


def test_criteo_kaggle_100_steps_overlapped():
    """configs[1], 100 steps, in the exact launch configuration bench.py times (fused
    lookup, F_TIMERS, device-resident inputs, overlapped streams)."""
    cfg = W.config("criteo_kaggle", world=1)
    st = W.gen_stream(cfg, 100)
    run_overlapped(st, fused=True, sample_rows=_touched_sample(st, 100, 20000, 1))


def test_avazu_100_steps_recorded():
    """configs[2] (22 tables, 9.4e6 rows, d 64, batch 16384, cache 10 %), 100 steps, every
    set exact per step, sampled host rows after the final flush."""
    cfg = W.config("avazu", world=1)
    st = W.gen_stream(cfg, 100)
    ages = []
    r = run_parity(st, sample_rows=_touched_sample(st, 100, 20000, 2), fused=True,
                   on_step=lambda s, got: ages.append(len(got["ageout"])))
    assert sum(ages) > 0
    r["fr"].close()


def test_freebase_shape_sampled():
    """configs[3] at its shape (Freebase: 86.1M entities + 14,824 relations, d 400, TransE,
    batch 2000, chunks of 200 negatives; host w 138 GB, G in HBM -- FRUGAL_F_NO_HOST_STATE),
    15 steps: dedup and every schedule set exact per step, losses within 1e-5, 5000 sampled
    touched rows (w and G, authoritative values) within 1e-5."""
    F = _F()
    cfg = W.config("freebase", world=1)
    st = W.gen_stream(cfg, 16)
    r = run_parity(st, steps=15, sample_rows=_touched_sample(st, 15, 5000, 3),
                   flags=F.F_RECORD | F.F_NO_HOST_STATE)
    r["fr"].close()


# ----------------------------------------------------------------------------- GPU scatter drain
def test_gpu_drain_recorded_tiny():
    """FRUGAL_F_GPU_DRAIN (the side drain scatters rows into the table from a kernel instead of
    packing them for the flushing threads): every set, the gate, losses and the whole table exact."""
    F = _F()
    st = W.gen_stream(tiny1(lookahead=4, age_out=2, batch=128), 80)
    r = run_parity(st, flags=F.F_RECORD | F.F_GPU_DRAIN, fused=True)
    assert r["exact"]
    r["fr"].close()


@pytest.mark.parametrize("fused", [False, True])
def test_gpu_drain_overlapped_tiny(fused):
    F = _F()
    st = W.gen_stream(tiny1(), 100)
    run_overlapped(st, fused=fused, flags=F.F_TIMERS | F.F_GPU_DRAIN, exact=True)


def test_gpu_drain_dynamic_cache():
    F = _F()
    cfg = tiny1(lookahead=4, age_out=3, cache_ratio=0.05)
    st = W.with_dynamic_hot(W.gen_stream(cfg, 60), epoch=7)
    r = run_parity(st, flags=F.F_RECORD | F.F_GPU_DRAIN)
    assert r["exact"]
    r["fr"].close()


def test_gpu_drain_criteo_kaggle_100_steps_overlapped():
    """configs[1] at full size, 100 steps, overlapped, with the GPU scatter drain."""
    F = _F()
    cfg = W.config("criteo_kaggle", world=1)
    st = W.gen_stream(cfg, 100)
    run_overlapped(st, fused=True, flags=F.F_TIMERS | F.F_GPU_DRAIN, sample_rows=_touched_sample(st, 100, 20000, 4))


def test_flushing_threads_counts_and_env():
    """The default drain (flushing threads) with 1 and 7 threads (uneven shares) and the
    N3 transition that waits for them, bit-exact (subprocess: threads are read at init)."""
    import subprocess
    import sys
    for th in ("1", "7"):
        code = ("import sys; sys.path.insert(0, '.');"
                "from tests.test_gpu_parity import run_parity, run_overlapped, tiny1; "
                "from paper_conf_asplos_xiezggl25_b200 import workload as W;"
                "st = W.gen_stream(tiny1(batch=128, lookahead=4, age_out=2), 50);"
                "r = run_parity(st); assert r['exact']; r['fr'].close();"
                "run_overlapped(W.with_dynamic_hot(st, epoch=7), exact=True); print('OK')")
        e = dict(os.environ, FRUGAL_FLUSH_THREADS=th)
        out = subprocess.run([sys.executable, "-c", code], env=e, capture_output=True, text=True,
                             cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))), timeout=600)
        assert "OK" in out.stdout, out.stdout + out.stderr


@pytest.mark.parametrize("fused", [False, True])
def test_host_inputs_e2e_path(fused):
    """The e2e leg's path: ids, x and y from pinned host memory through the C ABI (frugal_step
    copies the ids, frugal_dot_model copies x and y into its staging), ragged batches."""
    cfg = tiny1(batch=128, lookahead=4, age_out=2)
    rng = np.random.default_rng(41)
    counts = rng.integers(0, 129, size=(50, 1)).astype(np.int32)
    counts[6] = 0
    st = W.gen_stream(cfg, 50, counts=counts)
    run_overlapped(st, fused=fused, exact=True, host_inputs=True)


@pytest.mark.parametrize("env", [{}, {"FRUGAL_HOST_FLUSH": "0"}, {"FRUGAL_URGENT_SIDE": "0"}])
def test_host_table_contents_every_step(env):
    """The flushed BYTES, not only the flushed sets: after every step (all of the step's flushes
    applied -- urgent bucket, drain, age-outs, by the flushing threads or the GPU), the whole host
    table equals the oracle's simulated host table (each row = its value at its last flush),
    bit for bit.  Catches a flush that copies a row after the optimizer moved it (world 1 flushes
    the urgent bucket off the critical path from the source the scheduler recorded)."""
    import subprocess
    import sys
    code = ("import sys; sys.path.insert(0, '.'); import numpy as np;"
            "from tests.test_gpu_parity import tiny1; from oracle.oracle import Oracle;"
            "from paper_conf_asplos_xiezggl25_b200 import workload as W;"
            "from paper_conf_asplos_xiezggl25_b200.harness import Trainer, make_context;"
            "st = W.gen_stream(tiny1(batch=128, lookahead=4, age_out=2), 40);"
            "fr = make_context(st); tr = Trainer(fr, st, fused_lookup=True, device_inputs=True); o = Oracle(st);"
            "ks = np.arange(st.cfg.n_rows);"
            "[(tr.step(), o.step(), (lambda a, b: (np.array_equal(a[0], b[0]) or sys.exit(f'host w differs at step {s}')))"
            "  (fr.read_host(ks), o.host_rows(ks))) for s in range(st.steps)];"
            "print('OK')")
    e = dict(os.environ)
    e.update(env)
    out = subprocess.run([sys.executable, "-c", code], env=e, capture_output=True, text=True,
                         cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))), timeout=600)
    assert "OK" in out.stdout, out.stdout + out.stderr
