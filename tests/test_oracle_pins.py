"""Pins of the CPU oracle against things other than itself (CPU only).

Each test names the PAPER.md passage / closed form / brute force it pins.
"""
import dataclasses
import json
import math
import os

import numpy as np
import pytest

from oracle.oracle import (INF, Oracle, L_URGENT)
from paper_conf_asplos_xiezggl25_b200 import workload as W

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def tiny_random_stream(seed, world=2, steps=12, rows=40, batch=6, slots=1, alpha=0.9,
                       lookahead=3, age_out=3, cache_ratio=0.2, ragged=True, dim=4):
    cfg = W.WorkloadConfig("t", [rows] if slots == 1 else [rows] * slots, dim=dim, batch=batch,
                           world=world, alpha=alpha, lookahead=lookahead, age_out=age_out,
                           cache_ratio=cache_ratio, seed_ids=seed)
    rng = np.random.default_rng(seed + 100)
    counts = None
    if ragged:
        counts = rng.integers(0, batch + 1, size=(steps, world)).astype(np.int32)
    return W.gen_stream(cfg, steps, world, counts=counts)


# ----------------------------------------------------------------------------- init
def test_init_splitmix64_published_vector():
    """init(seed=0,k=0,j=0) uses splitmix64(0) = 0xE220A8397B1DCDAF (the published
    first output of SplitMix64 from state 0); u = top 24 bits / 2^24 (reading R18)."""
    cfg = W.config("tiny", seed_init=0)
    st = W.stream_from_lists(cfg, [[[1], [2]]])
    o = Oracle(st)
    u = 0xE220A8 / 2**24
    assert o.init_value(0, 0) == np.float32(np.float32(0.05) * np.float32(2 * u - 1))


# ----------------------------------------------------------------------------- dedup
@pytest.mark.parametrize("seed", range(6))
def test_dedup_brute_force(seed):
    st = tiny_random_stream(seed, slots=2)
    o = Oracle(st)
    for s in range(st.steps):
        for g in range(st.ids.shape[1]):
            m = int(st.counts[s, g]) * st.cfg.slots
            ids = st.ids[s, g, :m].tolist()
            uq, inv = o.dedup(s, g)
            assert uq.tolist() == sorted(set(ids))
            assert [uq[i] for i in inv] == ids


# ----------------------------------------------------------------------------- next access / readers
def _readers(st, k, t):
    F = st.cfg.slots
    return {g for g in range(st.ids.shape[1]) if k in st.ids[t, g, :st.counts[t, g] * F].tolist()}


@pytest.mark.parametrize("seed", range(4))
def test_next_access_brute_force(seed):
    st = tiny_random_stream(seed)
    L = st.cfg.lookahead
    o = Oracle(st)
    hot = set(st.hot.tolist())
    n = st.ids.shape[1]
    for k in range(st.cfg.n_rows):
        for u in range(st.steps):
            exp = INF
            for t in range(u + 1, min(u + L, st.steps - 1) + 1):
                if _readers(st, k, t):
                    exp = t
                    break
            assert o.next_access(k, u) == exp
            nh = any(not (g == k % n and k in hot) for g in _readers(st, k, u))
            assert o.needs_host(k, u) == nh


# ----------------------------------------------------------------------------- Fig. 6 golden trace
def test_fig6_golden_trace():
    gold = json.load(open(os.path.join(GOLD, "fig6.json")))
    cfg = W.WorkloadConfig("fig6", [8], dim=4, batch=2, world=gold["world"],
                           lookahead=gold["lookahead"], age_out=2, cache_ratio=0.0)
    st = W.stream_from_lists(cfg, gold["steps"])
    o = Oracle(st, hot=np.array(gold["hot"], dtype=np.int64))
    ex = gold["expect"]
    for k, u, nxt in ex["next"]:
        assert o.next_access(k, u) == (INF if nxt is None else nxt)
    for s in range(st.steps):
        assert o.step() == s
        sch = o.schedule()
        assert sch["gate_wait"] == ex["gate_wait"][s]
        assert sch["urgent"].tolist() == ex["urgent"][s]
        assert [[int(k), int(p)] for k, p in zip(sch["deferred"], sch["deferred_p"])] == ex["deferred"][s]
        if s < st.steps - 1:
            # k3 is held (INF) and not flushed before the end (L1084-1088)
            assert 3 in sch["inf"].tolist() or s == 0
    assert o.final_flush().tolist() == ex["final_flush"]
    assert o.violations == 0


# ----------------------------------------------------------------------------- invariant (2)
@pytest.mark.parametrize("seed", range(12))
def test_invariant_holds_random(seed):
    rng = np.random.default_rng(seed)
    L = int(rng.choice([2, 3, 5]))
    D = int(rng.choice([1, L, 2 * L]))
    st = tiny_random_stream(seed, world=int(rng.integers(1, 5)), lookahead=L, age_out=D,
                            cache_ratio=float(rng.choice([0.0, 0.1, 0.3])), steps=16)
    o = Oracle(st)
    o.run()
    assert o.violations == 0
    o.final_flush()
    # after the final flush the host table equals the synchronous values (w and G)
    ks = np.arange(st.cfg.n_rows)
    w, G = o.read_rows(ks)
    hw, hG = o.host_rows(ks)
    assert np.array_equal(w, hw) and np.array_equal(G, hG)


def test_invariant_negative_lost_urgent_flush():
    """Dropping one urgent flush must trip invariant (2) (L1104-1108)."""
    gold = json.load(open(os.path.join(GOLD, "fig6.json")))
    cfg = W.WorkloadConfig("fig6", [8], dim=4, batch=2, world=2, lookahead=2, cache_ratio=0.0)
    st = W.stream_from_lists(cfg, gold["steps"])
    o = Oracle(st, skip_urgent_step=1, hot=np.zeros(0, dtype=np.int64))
    o.run()
    assert o.violations > 0


# ----------------------------------------------------------------------------- literal P2F simulation
def literal_p2f(st, hot, L):
    """PAPER.md §3.3 literally: g-entries with R (future host-read steps from the
    L-step sample queue) and W (pending update steps); priority per Eq. (1);
    the gate of step s passes once every entry with priority <= s is flushed
    (lazy flushers).  Returns the set flushed at each gate."""
    n = st.ids.shape[1]
    S = st.steps
    R, Wset = {}, {}
    flushed = []

    def host_reads(t):
        out = set()
        for g in range(n):
            for k in st.ids[t, g, :st.counts[t, g] * st.cfg.slots].tolist():
                if not (g == k % n and k in hot):
                    out.add(k)
        return out

    def prio(k):
        if Wset.get(k) and R.get(k):
            return min(R[k])
        return INF

    for t in range(min(L - 1, S)):
        for k in host_reads(t):
            R.setdefault(k, set()).add(t)
    for s in range(S):
        t = s + L - 1
        if t < S:
            for k in host_reads(t):
                R.setdefault(k, set()).add(t)
        f = {k for k in Wset if Wset[k] and prio(k) <= s}
        for k in f:
            Wset[k] = []
        flushed.append(f)
        for k in host_reads(s):
            R[k].discard(s)
        touched = set()
        for g in range(n):
            touched |= set(st.ids[s, g, :st.counts[s, g] * st.cfg.slots].tolist())
        for k in touched:
            Wset.setdefault(k, []).append(s)
    return flushed


@pytest.mark.parametrize("seed", range(10))
def test_schedule_matches_literal_p2f(seed):
    rng = np.random.default_rng(1000 + seed)
    L = int(rng.choice([2, 3, 4]))
    st = tiny_random_stream(seed, world=int(rng.integers(1, 4)), lookahead=L, age_out=10**6,
                            cache_ratio=float(rng.choice([0.0, 0.2])), steps=14)
    hot = set(st.hot.tolist())
    lit = literal_p2f(st, hot, L)
    o = Oracle(st)
    by_deadline = {}
    for s in range(st.steps):
        o.step()
        sch = o.schedule()
        assert sch["ageout"].size == 0
        for k, p in zip(sch["deferred"].tolist(), sch["deferred_p"].tolist()):
            assert s < p <= s + L - 1
            by_deadline.setdefault(p, set()).add(k)
        mine = set(sch["urgent"].tolist()) | by_deadline.get(s, set())
        assert mine == lit[s], (s, mine, lit[s])
        assert sch["gate_wait"] == bool(sch["urgent"].size)
    assert o.violations == 0


@pytest.mark.parametrize("seed", range(6))
def test_schedule_with_ageout_brackets_literal(seed):
    """With age-out, U(s) ∪ deferred-due(s) ⊆ literal(s) ⊆ that ∪ rows aged out earlier."""
    rng = np.random.default_rng(2000 + seed)
    L = int(rng.choice([2, 3, 4]))
    st = tiny_random_stream(seed, world=int(rng.integers(1, 4)), lookahead=L, age_out=int(rng.integers(1, 4)),
                            cache_ratio=0.2, steps=16)
    lit = literal_p2f(st, set(st.hot.tolist()), L)
    o = Oracle(st)
    by_deadline, aged = {}, set()
    for s in range(st.steps):
        o.step()
        sch = o.schedule()
        for k, p in zip(sch["deferred"].tolist(), sch["deferred_p"].tolist()):
            by_deadline.setdefault(p, set()).add(k)
        mine = set(sch["urgent"].tolist()) | by_deadline.get(s, set())
        assert mine <= lit[s]
        assert lit[s] <= mine | aged
        aged |= set(sch["ageout"].tolist())
    assert o.violations == 0


# ----------------------------------------------------------------------------- model glue vs fp64 autograd
def test_glue_gradient_vs_torch_fp64():
    torch = pytest.importorskip("torch")
    cfg = W.WorkloadConfig("g", [30, 20, 10], dim=8, batch=5, world=2, cache_ratio=0.0)
    st = W.gen_stream(cfg, 3, counts=np.array([[5, 3], [4, 5], [0, 2]], dtype=np.int32))
    o = Oracle(st)
    for s in range(st.steps):
        ks = np.arange(cfg.n_rows)
        w0, _ = o.read_rows(ks)
        o.step()
        E = torch.tensor(w0, dtype=torch.float64, requires_grad=True)
        nb = int(st.counts[s].sum())
        loss = 0
        for g in range(2):
            c = int(st.counts[s, g])
            if c == 0:
                continue
            ids = torch.tensor(st.ids[s, g, :c * 3].reshape(c, 3))
            e = E[ids]                                      # [c, F, d]
            x = torch.tensor(st.x[s, g, :c], dtype=torch.float64)
            y = torch.tensor(st.y[s, g, :c], dtype=torch.float64)
            inter = torch.einsum("bfd,bgd->bfg", e, e)
            z = torch.triu(inter, diagonal=1).sum((1, 2)) + torch.einsum("bd,bfd->b", x, e)
            loss = loss + torch.nn.functional.binary_cross_entropy_with_logits(z, y, reduction="sum")
        (loss / nb).backward()
        assert abs(o.loss(s) - float(loss.detach()) / nb) < 1e-8  # S is summed in fp32 (R16)
        # per-position gradients of the oracle, summed per row = dL/dE
        acc = np.zeros_like(w0, dtype=np.float64)
        for g in range(2):
            c = int(st.counts[s, g])
            gr = o.grad(g)[:c * 3]
            np.add.at(acc, st.ids[s, g, :c * 3], gr.astype(np.float64))
        ref = E.grad.numpy()
        assert np.abs(acc - ref).max() <= 1e-6 * max(1e-3, np.abs(ref).max())


# ----------------------------------------------------------------------------- reduction vs dense one-hot
@pytest.mark.parametrize("seed", range(3))
def test_partials_vs_dense_onehot(seed):
    st = tiny_random_stream(seed, slots=2, batch=8, dim=6)
    o = Oracle(st)
    for s in range(4):
        o.step()
        for g in range(st.ids.shape[1]):
            m = int(st.counts[s, g]) * st.cfg.slots
            ids = st.ids[s, g, :m]
            gr = o.grad(g)[:m].astype(np.float64)
            keys, P = o.partial(g)
            A = np.zeros((m, st.cfg.n_rows))
            A[np.arange(m), ids] = 1.0
            dense = A.T @ gr
            assert keys.tolist() == sorted(set(ids.tolist()))
            np.testing.assert_allclose(P, dense[keys], rtol=1e-6, atol=1e-9)


# ----------------------------------------------------------------------------- optimizer closed forms
def test_adagrad_closed_form_single_row():
    """Linear loss <a, w>: grad = a each step ⇒ G_k = k a², w_s = w0 - lr Σ_k a/(√k |a| + eps)."""
    S = 60
    cfg = W.WorkloadConfig("a", [1], dim=4, batch=1, world=1, opt="adagrad", lr=0.05, cache_ratio=0.0)
    st = W.stream_from_lists(cfg, [[[0]]] * S)
    a = np.array([0.3, -0.02, 1.5, -7.0], dtype=np.float32)
    st.x[:] = a
    o = Oracle(st, model="const")
    w0, _ = o.read_rows([0])
    o.run()
    w, G = o.read_rows([0])
    a64 = a.astype(np.float64)
    k = np.arange(1, S + 1, dtype=np.float64)[:, None]
    exp_w = w0[0].astype(np.float64) - 0.05 * (a64[None, :] / (np.sqrt(k) * np.abs(a64)[None, :] + 1e-10)).sum(0)
    np.testing.assert_allclose(G[0], S * a64 ** 2, rtol=1e-5)
    np.testing.assert_allclose(w[0], exp_w, rtol=0, atol=2e-6)


def test_sgd_closed_form_l2():
    """L2 loss ½|w - t|² averaged over nb occurrences of one row: w_s = t + (1-lr)^s (w0 - t)."""
    S, lr = 25, 0.3
    cfg = W.WorkloadConfig("a", [1], dim=3, batch=4, world=2, opt="sgd", lr=lr, cache_ratio=0.0)
    st = W.stream_from_lists(cfg, [[[0, 0, 0], [0, 0]]] * S)
    t = np.array([0.5, -1.0, 2.0], dtype=np.float32)
    st.x[:] = t
    o = Oracle(st, model="l2")
    w0, _ = o.read_rows([0])
    o.run()
    w, _ = o.read_rows([0])
    exp = t + (1 - lr) ** S * (w0[0].astype(np.float64) - t)
    np.testing.assert_allclose(w[0], exp, rtol=0, atol=1e-6)


def test_adagrad_matches_torch_optim():
    torch = pytest.importorskip("torch")
    st = tiny_random_stream(3, world=2, slots=2, batch=8, dim=5, ragged=False)
    st.cfg.opt = "adagrad"
    o = Oracle(st)
    ks = np.arange(st.cfg.n_rows)
    w_prev, G_prev = o.read_rows(ks)
    param = torch.nn.Parameter(torch.tensor(w_prev))
    opt = torch.optim.Adagrad([param], lr=st.cfg.lr, eps=st.cfg.eps, initial_accumulator_value=0.0)
    for s in range(6):
        o.step()
        grad = np.zeros_like(w_prev)
        for g in range(2):
            keys, P = o.partial(g)
            grad[keys] += P
        param.grad = torch.tensor(grad)
        opt.step()
        w, _ = o.read_rows(ks)
        np.testing.assert_allclose(w, param.detach().numpy(), rtol=0, atol=2e-7)


def test_cross_world_equivalence_sgd():
    """Synchronous semantics: n=2 ranks == n=1 on the concatenated batch (Q14, within fp32 regrouping)."""
    st2 = tiny_random_stream(5, world=2, slots=2, batch=6, dim=4, ragged=False, steps=10)
    cfg1 = dataclasses.replace(st2.cfg, batch=12, world=1, opt="sgd", lr=1.0)
    st2.cfg.opt, st2.cfg.lr = "sgd", 1.0
    S = st2.steps
    st1 = W.Stream(cfg1, st2.ids.reshape(S, 1, -1).copy(), st2.counts.sum(1, keepdims=True).astype(np.int32),
                   st2.x.reshape(S, 1, 12, -1).copy(), st2.y.reshape(S, 1, 12).copy(), st2.hot)
    o1, o2 = Oracle(st1), Oracle(st2)
    o1.run(); o2.run()
    ks = np.arange(st2.cfg.n_rows)
    w1, _ = o1.read_rows(ks)
    w2, _ = o2.read_rows(ks)
    w0 = np.array([[o1.init_value(k, j) for j in range(4)] for k in ks], dtype=np.float32)
    assert np.abs(w1 - w0).max() > 1e-3        # non-vacuous
    np.testing.assert_allclose(w1, w2, rtol=0, atol=1e-6)
    for s in range(S):
        assert abs(o1.loss(s) - o2.loss(s)) < 1e-9


# ----------------------------------------------------------------------------- TransE glue (R26)
def test_transe_glue_vs_torch_fp64():
    """KG glue: TransE-L2 with chunked shared negatives -- loss and
    per-row gradients equal fp64 torch.autograd of the same objective."""
    torch = pytest.importorskip("torch")
    cfg = W.config("tiny_kg", batch=20, neg_chunk=8, dim=6, world=2, table_rows=[40, 5], alpha=0.5)
    st = W.gen_stream(cfg, 3, counts=np.array([[20, 13], [7, 20], [0, 20]], dtype=np.int32))
    o = Oracle(st)
    F, d = 4, cfg.dim
    for s in range(st.steps):
        ks = np.arange(cfg.n_rows)
        w0, _ = o.read_rows(ks)
        o.step()
        E = torch.tensor(w0, dtype=torch.float64, requires_grad=True)
        nb = int(st.counts[s].sum())
        loss = 0
        for g in range(2):
            cnt = int(st.counts[s, g])
            ids = torch.tensor(st.ids[s, g, :cnt * F].reshape(cnt, F))
            for b0 in range(0, cnt, cfg.neg_chunk):
                c = ids[b0:b0 + cfg.neg_chunk]
                h, r, t, neg = E[c[:, 0]], E[c[:, 1]], E[c[:, 2]], E[c[:, 3]]
                pos = cfg.gamma - torch.linalg.norm(h + r - t, dim=1)
                negs = cfg.gamma - torch.linalg.norm((h + r)[:, None, :] - neg[None, :, :], dim=2)
                loss = loss + torch.nn.functional.softplus(-pos).sum() + torch.nn.functional.softplus(negs).mean(1).sum()
        if nb == 0:
            continue
        (loss / nb).backward()
        assert abs(o.loss(s) - float(loss.detach()) / nb) < 1e-9 * max(1.0, abs(float(loss.detach())))
        acc = np.zeros_like(w0, dtype=np.float64)
        for g in range(2):
            cnt = int(st.counts[s, g])
            np.add.at(acc, st.ids[s, g, :cnt * F], o.grad(g)[:cnt * F].astype(np.float64))
        ref = E.grad.numpy()
        assert np.abs(acc - ref).max() <= 1e-6 * max(1e-3, np.abs(ref).max())


# ----------------------------------------------------------------------------- long segments (R23)
def _const_stream(seq, dim=4, world=1):
    """One step, one rank, slot 0 = row seq[b] for sample b; model 'const' makes the glue
    gradient of position b exactly x_b (oracle OR_MODEL_CONST: linear loss <x_b, e>)."""
    cfg = W.WorkloadConfig("seg", [max(seq) + 1], dim=dim, batch=len(seq), world=world,
                           lookahead=2, age_out=1, cache_ratio=0.0)
    return W.stream_from_lists(cfg, [[list(seq)]])


@pytest.mark.parametrize("n", [1, 63, 64, 65, 127, 128, 129, 1000, 1537])
def test_partials_long_segments_exact_integers(n):
    """Partial of a row with n occurrences (up to 1537: 25 chunks of the R23 chunked
    order, ragged last chunk) when every gradient is a small integer: the fp32 sum is
    then exact in ANY order, so the oracle's partial must equal the integer sum bit for
    bit (a dropped, repeated or mis-indexed occurrence anywhere changes it).  Rows with
    1 and 2 occurrences sit beside it (neighbouring segments must not bleed in)."""
    rng = np.random.default_rng(n)
    seq = [0] * n + [1] + [2, 2]
    rng.shuffle(seq)
    st = _const_stream(seq)
    x = rng.integers(-4, 5, size=(len(seq), 4)).astype(np.float32)
    x[x == 0] = 3.0                    # no zero term: every dropped occurrence shows
    st.x[0, 0, :len(seq)] = x
    o = Oracle(st, model="const")
    o.step()
    keys, P = o.partial(0)
    assert keys.tolist() == [0, 1, 2]
    for r in range(3):
        exact = x[np.array(seq) == r].astype(np.int64).sum(0)
        assert np.array_equal(P[r], exact.astype(np.float32)), (r, P[r], exact)


def test_partials_long_segment_error_bound():
    """Random fp32 gradients, 1500 occurrences of one row: |P - exact| <= (64 + n/64) u sum|g|
    (the textbook bound of a two-level sequential sum with chunks of 64, u = 2^-24; the exact
    value is the fp64 sum of the same fp32 terms)."""
    rng = np.random.default_rng(7)
    n = 1500
    seq = [0] * n + [1] * 5
    rng.shuffle(seq)
    st = _const_stream(seq)
    x = rng.normal(0, 1, size=(len(seq), 4)).astype(np.float32)
    st.x[0, 0, :len(seq)] = x
    o = Oracle(st, model="const")
    o.step()
    keys, P = o.partial(0)
    g = x[np.array(seq) == 0].astype(np.float64)
    exact = g.sum(0)
    bound = (64 + n / 64 + 2) * 2.0 ** -24 * np.abs(g).sum(0)
    assert np.all(np.abs(P[0] - exact) <= bound), (np.abs(P[0] - exact), bound)


def test_partials_chunk_order_R23_hand_value():
    """Reading R23 fixed by a hand-derived value.  Row 0 occurs 128 times: position 0
    carries 1.0, the other 127 carry 2^-25 = half an ulp of 1.0, so each is lost when added to
    1.0 (round to nearest, ties to even) but sums exactly with its peers.  Chunks of 64:
    chunk 0 = 1.0 (its 63 small terms round away one by one), chunk 1 = 64 * 2^-25 = 2^-19
    (exact), total 1 + 2^-19.  A plain sequential sum would give 1.0, chunks of 32 give
    1 + 3*2^-20, chunks of 128 or 256 give 1.0."""
    seq = [0] * 128
    st = _const_stream(seq, dim=4)
    x = np.full((128, 4), 2.0 ** -25, dtype=np.float32)
    x[0] = 1.0
    st.x[0, 0, :128] = x
    o = Oracle(st, model="const")
    o.step()
    _, P = o.partial(0)
    assert np.all(P[0] == np.float32(1.0 + 2.0 ** -19)), P[0]


# ----------------------------------------------------------------------------- age-out (R9)
def _trace(per_step, L, D, hot=()):
    cfg = W.WorkloadConfig("age", [64], dim=4, batch=4, world=1, lookahead=L, age_out=D, cache_ratio=0.0)
    st = W.stream_from_lists(cfg, per_step)
    o = Oracle(st, hot=np.array(sorted(hot), dtype=np.int64))
    out = []
    for s in range(st.steps):
        o.step()
        sch = o.schedule()
        out.append(dict(age=sch["ageout"].tolist(), urgent=sch["urgent"].tolist(),
                        deferred=sorted(zip(sch["deferred"].tolist(), sch["deferred_p"].tolist())),
                        inf=sch["inf"].tolist()))
    assert o.violations == 0
    return out, o


@pytest.mark.parametrize("D", [1, 2, 3, 5])
def test_ageout_hand_trace(D):
    """Reading R9 (a row with no read in sight is held, then
    flushed by the lazy flushers): a cold row updated at step u and never read again gets
    priority INF from the scheduler of u+1 and is flushed by the age-out of step u+1+D --
    exactly D steps after the scheduler that found no read in its window.  Row 10+u is read
    only at step u (one filler row per step), so the age-out set of step s is exactly
    {10 + (s-1-D)} for s >= 1+D and empty before; the INF set of step s holds the rows
    updated at s-1-D+1 .. s-1."""
    S, L = 12, 3
    per_step = [[[10 + s]] for s in range(S)]
    out, o = _trace(per_step, L, D)
    for s in range(S):
        exp_age = [10 + (s - 1 - D)] if s >= 1 + D else []
        assert out[s]["age"] == exp_age, (s, out[s]["age"], exp_age)
        assert out[s]["urgent"] == [] and out[s]["deferred"] == []
        exp_inf = [10 + u for u in range(max(0, s - D), s)]
        assert out[s]["inf"] == exp_inf, (s, out[s]["inf"], exp_inf)
    # the last scheduler (step S-1) ages out u <= S-2-D: rows updated at S-1-D .. S-1 are
    # still dirty and go out with the final flush
    assert o.final_flush().tolist() == [10 + u for u in range(S - 1 - D, S)]


def test_ageout_vs_adjust_priority_hand_trace():
    """Hand trace of the two ways an INF row leaves INF (R9 vs Fig. 6 step 4, L1074-1077).
    L = 3.  Row 7 is read at steps 0 and 5; rows 20+s fill every step.
      D = 10: step 1 buckets row 7 INF (no read in [1, 3]); the ingest of step 3+3-1 = 5
      (AdjustPriority, made by frugal_step(3)) gives it deadline 5: D(3) = {(7, 5)}; never
      aged out.
      D = 1: row 7 is aged out by step 0+1+1 = 2, before the read of step 5 enters the
      window; at step 3 it is clean, so no AdjustPriority, no deferred entry."""
    per_step = [[[20, 7]], [[21]], [[22]], [[23]], [[24]], [[25, 7]], [[26]], [[27]]]
    out, _ = _trace(per_step, 3, 10)
    assert (7, 5) in out[3]["deferred"]
    assert all(7 not in out[s]["age"] for s in range(len(per_step)))
    assert all((7, 5) not in out[s]["deferred"] for s in range(len(per_step)) if s != 3)
    out, _ = _trace(per_step, 3, 1)
    assert 7 in out[2]["age"]
    assert all(k != 7 for s in range(len(per_step)) for k, _ in out[s]["deferred"])
    assert [s for s in range(len(per_step)) if 7 in out[s]["age"]] == [2, 7]  # then re-aged after the update at 5


def test_ageout_skips_hot_rows():
    """R9: hot (cached) rows with no host-reader are never aged out (they stay dirty until a
    host-reader appears or the final flush).  Row 3 hot, read at step 0 only, D = 1."""
    per_step = [[[3, 30]], [[31]], [[32]], [[33]], [[34]]]
    out, o = _trace(per_step, 2, 1, hot={3})
    assert all(3 not in out[s]["age"] for s in range(5))
    assert 3 in o.final_flush().tolist()


def test_hot_flush_moves_w_only_R8():
    """Reading R8 by hand: an owner's hot row flushed during training for another rank's read
    moves w only (its Adagrad state G stays with the owner until the final flush); a cold row
    moves w and G.  world 2, no age-out in sight (D = 10), L = 2; rows 0 (hot) and 2 (cold)
    are owned by rank 0.  Step 0: rank 0 reads 0 and 2.  Step 1: rank 1 reads 0 and 2, so
    both are urgent at step 1 (U(1) = {0, 2}) and the host copies hold their post-step-0
    values.  G of row 0 on the host is then still G0 = 0; G of row 2 is g0^2 != 0."""
    cfg = W.WorkloadConfig("r8", [8], dim=4, batch=2, world=2, lookahead=2, age_out=10, cache_ratio=0.0)
    st = W.stream_from_lists(cfg, [[[0, 2], []], [[], [0, 2]], [[], []]])
    o = Oracle(st, hot=np.array([0], dtype=np.int64))
    o.step()
    w0, G0 = o.read_rows([0, 2])  # values after step 0
    o.step()
    assert o.schedule()["urgent"].tolist() == [0, 2]
    hw, hG = o.host_rows([0, 2])
    assert np.array_equal(hw, w0)
    assert np.all(G0 > 0)
    assert np.all(hG[0] == 0.0) and np.array_equal(hG[1], G0[1])
    o.step()
    o.final_flush()
    w, G = o.read_rows([0, 2])
    hw, hG = o.host_rows([0, 2])
    assert np.array_equal(hw, w) and np.array_equal(hG, G)
