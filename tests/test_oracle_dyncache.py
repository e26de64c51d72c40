"""Pins of the oracle's N3 dynamic cache (reading R27), CPU only.

What pins it, besides itself:
* synchronous semantics (proof §3.3): the values (tables,
  losses) cannot depend on which rows are cached -- bit-identical to the static-cache run;
* invariant (2) (L1104-1108) at every host read, now against the hot set of the step;
* the literal P2F model of §3.3 (R/W sets, Eq. (1), gate "top > s") with the hot set of
  each step: U(s) ∪ deferred-due(s) ⊆ literal(s) ⊆ that ∪ rows aged out or flushed by a
  transition earlier;
* a hand-derived trace (below) and a negative test (a lost transition flush trips (2)).
"""
import numpy as np
import pytest

from oracle.oracle import INF, Oracle
from paper_conf_asplos_xiezggl25_b200 import workload as W

from .test_oracle_pins import tiny_random_stream


def random_dyn_stream(seed, steps=24):
    rng = np.random.default_rng(5000 + seed)
    L = int(rng.choice([2, 3, 4]))
    D = int(rng.choice([1, L, 2 * L]))
    E = int(rng.integers(L + 1, L + 4))
    st = tiny_random_stream(seed, world=int(rng.integers(1, 4)), lookahead=L, age_out=D,
                            cache_ratio=float(rng.choice([0.1, 0.3])), steps=steps)
    # random hot sets (not frequency-based) stress every kind of turnover
    sched = []
    for t0 in range(E, steps, E):
        k = int(rng.integers(0, st.cfg.n_rows // 2))
        sched.append((t0, np.sort(rng.choice(st.cfg.n_rows, size=k, replace=False)).astype(np.int64)))
    return st, W.dataclasses.replace(st, hot_schedule=sched), L


@pytest.mark.parametrize("seed", range(10))
def test_values_do_not_depend_on_the_cache(seed):
    st, dyn, _ = random_dyn_stream(seed)
    a, b = Oracle(st), Oracle(dyn)
    a.run()
    b.run()
    assert a.violations == 0 and b.violations == 0
    ks = np.arange(st.cfg.n_rows)
    wa, Ga = a.read_rows(ks)
    wb, Gb = b.read_rows(ks)
    assert np.array_equal(wa, wb) and np.array_equal(Ga, Gb)
    assert [a.loss(s) for s in range(st.steps)] == [b.loss(s) for s in range(st.steps)]
    b.final_flush()
    hw, hG = b.host_rows(ks)
    assert np.array_equal(hw, wb) and np.array_equal(hG, Gb)


def literal_p2f_dyn(st, L):
    """PAPER.md §3.3 literally (as tests/test_oracle_pins.literal_p2f), with the host-read
    classification of step t against the hot set in force at t."""
    n, S, F = st.ids.shape[1], st.steps, st.cfg.slots
    epochs = [(0, set(st.hot.tolist()))] + [(t0, set(np.asarray(h).tolist())) for t0, h in st.hot_schedule]

    def hot_at(t):
        return [h for t0, h in epochs if t0 <= t][-1]

    def host_reads(t):
        hot = hot_at(t)
        return {k for g in range(n) for k in st.ids[t, g, :st.counts[t, g] * F].tolist()
                if not (g == k % n and k in hot)}

    R, Wset, flushed = {}, {}, []
    for t in range(min(L - 1, S)):
        for k in host_reads(t):
            R.setdefault(k, set()).add(t)
    for s in range(S):
        t = s + L - 1
        if t < S:
            for k in host_reads(t):
                R.setdefault(k, set()).add(t)
        prio = {k: (min(R[k]) if Wset[k] and R.get(k) else INF) for k in Wset}
        f = {k for k in Wset if Wset[k] and prio[k] <= s}
        for k in f:
            Wset[k] = []
        flushed.append(f)
        for k in host_reads(s):
            R[k].discard(s)
        for g in range(n):
            for k in st.ids[s, g, :st.counts[s, g] * F].tolist():
                Wset.setdefault(k, []).append(s)
    return flushed


@pytest.mark.parametrize("seed", range(10))
def test_schedule_brackets_literal_p2f_with_dynamic_hot(seed):
    _, dyn, L = random_dyn_stream(seed)
    lit = literal_p2f_dyn(dyn, L)
    o = Oracle(dyn)
    by_deadline, early = {}, set()
    for s in range(dyn.steps):
        o.step()
        sch = o.schedule()
        for k, p in zip(sch["deferred"].tolist(), sch["deferred_p"].tolist()):
            assert s < p <= s + L - 1
            by_deadline.setdefault(p, set()).add(k)
        early |= set(sch["transition"].tolist())
        mine = set(sch["urgent"].tolist()) | by_deadline.get(s, set())
        assert mine <= lit[s], (s, mine - lit[s])
        assert lit[s] <= mine | early, (s, lit[s] - mine - early)
        early |= set(sch["ageout"].tolist())
    assert o.violations == 0


def test_transition_is_the_dirty_hotness_changes():
    """X(t0) = rows whose hotness changes at t0 and that are dirty when step t0 begins."""
    for seed in range(8):
        st, dyn, _ = random_dyn_stream(seed)
        bounds = {t0: set(np.asarray(h).tolist()) for t0, h in dyn.hot_schedule}
        hot = set(dyn.hot.tolist())
        o = Oracle(dyn)
        for s in range(dyn.steps):
            if s in bounds:
                new = bounds[s]
                want = sorted(k for k in hot ^ new if o.row_state(k) != 0)
                o.step()
                assert o.schedule()["transition"].tolist() == want
                hot = new
            else:
                o.step()
                assert o.schedule()["transition"].size == 0


def hand_trace():
    """world 1, L = 2, D = 10, rows 0..3; H = {1} until step 2, H' = {2} from t0 = 3.
    steps: 0: [1, 2]   1: [1]   2: [0]   3: [1, 2]   4: [2]
    s1: k1 (updated 0) next read 1, owner-only hot -> EXEMPT; k2 (updated 0) no read in
        [1, 2] -> INF.
    s2: k1 (updated 1) next read 3, cold there (H') -> deferred D(2) = {(1, 3)};
        AdjustPriority for t = 3: k2 INF, read at 3 only by its owner, hot there -> EXEMPT.
    s3 = t0: k1 leaves the cache clean (flushed at s2); k2 enters dirty (EXEMPT) -> X(3) = {2}.
    s4: k2 (updated 3, hot) read at 4 by its owner only -> EXEMPT; nothing urgent."""
    cfg = W.WorkloadConfig("dyn", [4], dim=4, batch=2, world=1, lookahead=2, age_out=10, cache_ratio=0.0)
    st = W.stream_from_lists(cfg, [[[1, 2]], [[1]], [[0]], [[1, 2]], [[2]]])
    st = W.dataclasses.replace(st, hot=np.array([1], np.int64),
                               hot_schedule=[(3, np.array([2], np.int64))])
    return st


def test_hand_trace():
    st = hand_trace()
    o = Oracle(st)
    got = []
    for s in range(st.steps):
        o.step()
        sch = o.schedule()
        got.append((sch["urgent"].tolist(), list(zip(sch["deferred"].tolist(), sch["deferred_p"].tolist())),
                    sch["transition"].tolist(), sch["exempt"].tolist(), sch["inf"].tolist()))
    assert got[1][3] == [1] and got[1][4] == [2]
    assert got[2][1] == [(1, 3)] and 2 in got[2][3]
    assert got[3][2] == [2]
    assert all(g[0] == [] for g in got)
    assert [g[2] for g in got] == [[], [], [], [2], []]
    assert o.violations == 0


def test_lost_transition_flush_trips_the_invariant():
    """An EVICTED row that is dirty at t0 and read at t0: its owner now reads it from the
    host, so losing its transition flush must trip invariant (2) (L1104-1108)."""
    cfg = W.WorkloadConfig("dyn", [4], dim=4, batch=2, world=1, lookahead=2, age_out=10, cache_ratio=0.0)
    # k1 hot until 2, read (and updated) by its owner at every step; evicted at t0 = 3
    st = W.stream_from_lists(cfg, [[[1]], [[1]], [[1]], [[1]]])
    st = W.dataclasses.replace(st, hot=np.array([1], np.int64), hot_schedule=[(3, np.array([2], np.int64))])
    ok = Oracle(st)
    ok.run()
    assert ok.violations == 0
    ok2 = Oracle(st)
    for _ in range(4):
        ok2.step()
    assert ok2.schedule()["transition"].tolist() == [1]
    bad = Oracle(st, skip_urgent_step=3)
    bad.run()
    assert bad.violations > 0
