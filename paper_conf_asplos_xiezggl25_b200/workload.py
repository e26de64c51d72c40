"""Seeded synthetic workload generator (ID streams, labels, dense features, hot set).

This module is the ONLY code shared by the CPU oracle (``oracle/``) and the CUDA
path: it produces *inputs* and holds none of the method's arithmetic (no dedup,
no next-access, no bucketing, no optimizer).  Both sides consume exactly the
arrays it returns.

Workload recipe (DESIGN.md §"Input recipe"):

* Embedding lookups follow PAPER.md §4.1 "Synthetic workloads" (L1273-1281):
  Zipfian keys with skew 0.9 / 0.99 (uniform = skew 0).  Each slot f reads table
  f; within a table, popularity rank r in [1, N_f] is drawn with
  P(r) ∝ r^-alpha by exact rejection-inversion sampling (Hörmann & Derflinger),
  and mapped to a local row id by a seeded Feistel bijection on [0, N_f) so the
  Zipf head is scattered over the id space.  The global row
  id is table_offset[f] + local id.
* Table shapes follow PAPER.md Table 2 (L1250-1263) as restated by BASELINE.json
  configs: Criteo-Kaggle (26 tables, 33,762,577 rows, d=32), Avazu-shaped
  (22 tables, ~9.4e6 rows, d=64), CriteoTB-shaped (Kaggle profile scaled to
  ~8.8e8 rows, d=128), plus the tiny 1-table config.
* Labels: planted y = [sum_f h(id_f) > 0] with h = +-1 from a hash of the id
  (SURVEY §8(c) Q15).  KG workloads (TransE, §4.1): samples are
  triples (h, r, t) plus one corrupting entity "neg" per triple; the negatives of a
  chunk of neg_chunk triples are shared by the chunk (DGL-KE chunked negative sampling,
  "negative sampling batch size of 200").  Entities and relations are Zipf(alpha).  Dense features x_b ~ N(0, 0.1^2) in R^d, frozen (they
  stand in for DLRM's bottom-MLP output).
* Hot (cached) set: the top floor(cache_ratio * N_f) rows of each table by
  frequency over the first min(S, 50) steps of the stream, ties broken by the
  smaller id ("5% of the total parameters", L1404-1406).
"""
from __future__ import annotations

import dataclasses
import math
from typing import List, Optional

import numpy as np

# Criteo Kaggle per-feature cardinalities (DLRM preprocessing); sum = 33,762,577
# which matches PAPER.md Table 2 "Criteo 26 34 M" (L1259).
CRITEO_KAGGLE_ROWS = [1460, 583, 10131227, 2202608, 305, 24, 12517, 633, 3, 93145,
                      5683, 8351593, 3194, 27, 14992, 5461306, 10, 5652, 2173, 4,
                      7046547, 18, 15, 286181, 105, 142572]
# Avazu-shaped: 22 fields (Table 2), ~9.4e6 ids (BASELINE.json config 3):
# two large fields plus 20 small ones (illustrative profile; the real per-field
# cardinalities are not in the paper).
AVAZU_ROWS = [6_700_000, 2_700_000, 240, 7, 7, 4737, 7745, 26, 8552, 559, 36,
              2686, 6729, 5, 4, 2626, 8, 9, 435, 4, 68, 172]


@dataclasses.dataclass
class WorkloadConfig:
    name: str
    table_rows: List[int]
    dim: int
    batch: int               # B per rank (per GPU); global batch = world * B (Q19)
    world: int = 1
    alpha: float = 0.9       # Zipf skew (0 = uniform)
    cache_ratio: float = 0.05
    lookahead: int = 10      # L
    age_out: int = 10        # D
    opt: str = "adagrad"     # "adagrad" | "sgd"
    lr: float = 0.05
    eps: float = 1e-10
    init_accum: float = 0.0
    init_scale: float = 0.05
    seed_ids: int = 1
    seed_labels: int = 2
    seed_init: int = 3
    seed_dense: int = 4
    # slot f reads table slot_tables[f] (None: slot f reads table f).  KG workloads use
    # slots (h, r, t, neg) -> tables (entities, relations, entities, entities).
    slot_tables: Optional[List[int]] = None
    model: str = "dot"       # "dot" (REC glue, R15) | "transe" (KG glue, R26)
    neg_chunk: int = 200     # TransE: negatives shared by chunks of this many triples (L1287-1288)
    gamma: float = 12.0      # TransE margin (DGL-KE default)

    @property
    def slots(self) -> int:
        return len(self.slot_tables) if self.slot_tables is not None else len(self.table_rows)

    def slot_table(self, f: int) -> int:
        return self.slot_tables[f] if self.slot_tables is not None else f

    @property
    def n_rows(self) -> int:
        return int(sum(self.table_rows))

    @property
    def table_offsets(self) -> np.ndarray:
        return np.concatenate([[0], np.cumsum(self.table_rows)[:-1]]).astype(np.int64)


def criteo_tb_rows(total: float = 8.8e8) -> List[int]:
    """CriteoTB-shaped tables: the Criteo-Kaggle cardinality profile scaled to `total` rows
    (Table 2: 882M rows at full size)."""
    scale = total / sum(CRITEO_KAGGLE_ROWS)
    return [max(1, int(round(r * scale))) for r in CRITEO_KAGGLE_ROWS]


def config(name: str, **over) -> WorkloadConfig:
    """The BASELINE.json configs restated as synthetic inputs.  criteo_tb takes
    `rows_total` (default 8.8e8) to scale its tables to what the host's memory holds."""
    if name == "tiny":          # configs[0]
        c = WorkloadConfig("tiny", [10_000], dim=16, batch=256, world=2)
    elif name == "criteo_kaggle":  # configs[1]
        c = WorkloadConfig("criteo_kaggle", list(CRITEO_KAGGLE_ROWS), dim=32, batch=8192, world=8)
    elif name == "avazu":       # configs[2]
        c = WorkloadConfig("avazu", list(AVAZU_ROWS), dim=64, batch=16384, world=8, cache_ratio=0.10)
    elif name == "freebase":    # configs[3]: Freebase-shaped KG (Table 2: 86.1M entities, 14.8K relations)
        c = WorkloadConfig("freebase", [86_100_000, 14_824], dim=400, batch=2000, world=8,
                           slot_tables=[0, 1, 0, 0], model="transe", neg_chunk=200)
    elif name == "fb15k":       # FB15k-shaped KG (Table 2, columns read as 15k entities, 1.3k relations)
        c = WorkloadConfig("fb15k", [14_951, 1_345], dim=400, batch=1200, world=8,
                           slot_tables=[0, 1, 0, 0], model="transe", neg_chunk=200)
    elif name == "tiny_kg":     # small KG case for parity tests
        c = WorkloadConfig("tiny_kg", [5_000, 40], dim=16, batch=96, world=1, slot_tables=[0, 1, 0, 0],
                           model="transe", neg_chunk=32, lookahead=4, age_out=3)
    elif name == "criteo_tb":   # configs[4]
        rows = criteo_tb_rows(over.pop("rows_total", 8.8e8))
        c = WorkloadConfig("criteo_tb", rows, dim=128, batch=8192, world=8, cache_ratio=0.10,
                           opt="sgd", lr=1.0)
    else:
        raise KeyError(name)
    return dataclasses.replace(c, **over)


# ----------------------------------------------------------------------------- Zipf sampler
def zipf_ranks(rng: np.random.Generator, n: int, alpha: float, size: int) -> np.ndarray:
    """Exact discrete Zipf on {1..n}, P(r) ∝ r^-alpha, by rejection-inversion.

    (Hörmann & Derflinger 1996, the algorithm used by Apache Commons'
    RejectionInversionZipfSampler.)  alpha == 0 gives the uniform distribution.
    Returns int64 ranks in [1, n].
    """
    if n == 1:
        return np.ones(size, dtype=np.int64)
    if alpha == 0.0:
        return rng.integers(1, n + 1, size=size, dtype=np.int64)
    a = float(alpha)

    def H(x):  # integral of x^-a, shifted so H(1) = 0
        lx = np.log(x)
        t = (1.0 - a) * lx
        # helper2: (exp(t)-1)/t, stable near 0
        return np.where(np.abs(t) > 1e-8, np.expm1(t) / np.where(t == 0, 1, t), 1.0 + t / 2.0) * lx

    def H_inv(y):
        t = y * (1.0 - a)
        t = np.maximum(t, -1.0 + 1e-16)
        # helper1: log1p(t)/t, stable near 0
        h1 = np.where(np.abs(t) > 1e-8, np.log1p(t) / np.where(t == 0, 1, t), 1.0 - t / 2.0)
        return np.exp(h1 * y)

    def h(x):
        return np.exp(-a * np.log(x))

    hx1 = float(H(np.array(1.5))) - 1.0
    hn = float(H(np.array(n + 0.5)))
    s = 2.0 - float(H_inv(np.array(H(np.array(2.5)) - h(np.array(2.0)))))
    out = np.empty(size, dtype=np.int64)
    todo = np.arange(size)
    while todo.size:
        u = hn + rng.random(todo.size) * (hx1 - hn)
        x = H_inv(u)
        k = np.clip(np.floor(x + 0.5), 1, n)
        acc = (k - x <= s) | (u >= H(k + 0.5) - h(k))
        out[todo[acc]] = k[acc].astype(np.int64)
        todo = todo[~acc]
    return out


def feistel_permute(x: np.ndarray, n: int, key: int) -> np.ndarray:
    """Seeded bijection on [0, n): 4-round balanced Feistel with cycle walking."""
    x = np.asarray(x, dtype=np.uint64).copy()
    if n <= 1:
        return x.astype(np.int64)
    bits = max(2, int(math.ceil(math.log2(n))))
    bits += bits & 1
    half = bits // 2
    mask = np.uint64((1 << half) - 1)
    keys = [np.uint64((key * 0x9E3779B97F4A7C15 + r * 0xBF58476D1CE4E5B9) & 0xFFFFFFFFFFFFFFFF)
            for r in range(4)]

    def rnd(v, k):
        z = (v ^ k) * np.uint64(0x94D049BB133111EB)
        z ^= z >> np.uint64(29)
        z *= np.uint64(0xBF58476D1CE4E5B9)
        z ^= z >> np.uint64(32)
        return z & mask

    todo = np.arange(x.size)
    with np.errstate(over="ignore"):
        while todo.size:
            v = x[todo]
            l, r = v >> np.uint64(half), v & mask
            for k in keys:
                l, r = r, l ^ rnd(r, k)
            v = (l << np.uint64(half)) | r
            x[todo] = v
            todo = todo[v >= np.uint64(n)]
    return x.astype(np.int64)


def _hash_sign(ids: np.ndarray, seed: int) -> np.ndarray:
    z = ids.astype(np.uint64) ^ np.uint64(seed * 0x2545F4914F6CDD1D & 0xFFFFFFFFFFFFFFFF)
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(33))) * np.uint64(0xFF51AFD7ED558CCD)
        z = (z ^ (z >> np.uint64(33))) * np.uint64(0xC4CEB9FE1A85EC53)
        z ^= z >> np.uint64(33)
    return np.where((z & np.uint64(1)) == 1, 1, -1).astype(np.int64)


@dataclasses.dataclass
class Stream:
    """A seeded ID stream: ids[S][world][batch*slots] (global row ids, position
    i = b*slots + f), counts[S][world] samples per rank, x[S][world][batch][dim],
    y[S][world][batch], and the hot set (sorted global ids)."""
    cfg: WorkloadConfig
    ids: np.ndarray
    counts: np.ndarray
    x: np.ndarray
    y: np.ndarray
    hot: np.ndarray
    # N3 dynamic cache (reading R27): [(t0, hot ids)], the hot set in force from step t0 on
    hot_schedule: list = dataclasses.field(default_factory=list)
    # host-table layout (frugal_config.host_order): global ids in host-slot order, or None
    host_order: Optional[np.ndarray] = None

    @property
    def steps(self) -> int:
        return self.ids.shape[0]


def gen_ids(cfg: WorkloadConfig, steps: int, world: Optional[int] = None) -> np.ndarray:
    world = cfg.world if world is None else world
    rng = np.random.default_rng(cfg.seed_ids)
    F, B = cfg.slots, cfg.batch
    offs = cfg.table_offsets
    ids = np.empty((steps, world, B, F), dtype=np.int64)
    for s in range(steps):
        for f in range(F):
            tb = cfg.slot_table(f)
            nf = cfg.table_rows[tb]
            r = zipf_ranks(rng, nf, cfg.alpha, world * B) - 1
            local = feistel_permute(r, nf, cfg.seed_ids * 1000003 + tb)
            ids[s, :, :, f] = (offs[tb] + local).reshape(world, B)
    return ids.reshape(steps, world, B * F)


def hot_set(cfg: WorkloadConfig, ids: np.ndarray, counts: Optional[np.ndarray] = None,
            window: int = 50) -> np.ndarray:
    """Top floor(ratio*N_f) rows per table by frequency over the first min(S, window) steps."""
    S = min(ids.shape[0], window)
    F, B = cfg.slots, cfg.batch
    sub = ids[:S].reshape(S, -1, B, F)
    if counts is not None:
        valid = np.arange(B)[None, None, :] < counts[:S, :, None]
    else:
        valid = np.ones(sub.shape[:3], dtype=bool)
    offs = cfg.table_offsets
    hot = []
    for f, nf in enumerate(cfg.table_rows):
        k = int(math.floor(cfg.cache_ratio * nf))
        if k <= 0:
            continue
        cols = [sub[:, :, :, q][valid] - offs[f] for q in range(F) if cfg.slot_table(q) == f]
        freq = np.bincount(np.concatenate(cols), minlength=nf)
        # sort by (-freq, id): stable argsort of -freq keeps smaller ids first
        order = np.argsort(-freq, kind="stable")[:k]
        hot.append(offs[f] + order)
    if not hot:
        return np.zeros(0, dtype=np.int64)
    return np.sort(np.concatenate(hot)).astype(np.int64)


def host_order(cfg: WorkloadConfig, ids: np.ndarray, counts: Optional[np.ndarray] = None) -> np.ndarray:
    """Host-table layout from past traffic: every row read in `ids` (steps of
    all ranks), most frequent first, ties by smaller id.  Rows never read are left to the
    library (they follow in id order).  A layout only moves bytes; no result depends on it."""
    S, world = ids.shape[0], ids.shape[1]
    F, B = cfg.slots, ids.shape[2] // cfg.slots
    sub = ids.reshape(S, world, B, F)
    if counts is not None:
        sub = sub[np.arange(B)[None, None, :] < counts[:, :, None]]
    freq = np.bincount(sub.ravel(), minlength=cfg.n_rows)
    seen = np.flatnonzero(freq)
    return seen[np.argsort(-freq[seen], kind="stable")].astype(np.int64)


def gen_stream(cfg: WorkloadConfig, steps: int, world: Optional[int] = None,
               counts: Optional[np.ndarray] = None) -> Stream:
    world = cfg.world if world is None else world
    ids = gen_ids(cfg, steps, world)
    if counts is None:
        counts = np.full((steps, world), cfg.batch, dtype=np.int32)
    counts = np.asarray(counts, dtype=np.int32)
    F, B, d = cfg.slots, cfg.batch, cfg.dim
    # padding positions beyond counts are zeroed (never read by either side)
    valid = (np.arange(B)[None, None, :] < counts[:, :, None])
    ids = ids.reshape(steps, world, B, F)
    ids[~valid] = 0
    ids = ids.reshape(steps, world, B * F)
    sgn = _hash_sign(ids, cfg.seed_labels).reshape(steps, world, B, F).sum(-1)
    y = (sgn > 0).astype(np.float32)
    y[~valid] = 0
    rng = np.random.default_rng(cfg.seed_dense)
    x = (rng.standard_normal((steps, world, B, d), dtype=np.float32) * np.float32(0.1)).astype(np.float32)
    x[~valid] = 0
    hot = hot_set(cfg, ids, counts)
    return Stream(cfg, np.ascontiguousarray(ids), counts, x, y, hot)


def with_dynamic_hot(st: Stream, epoch: int, window: Optional[int] = None) -> Stream:
    """N3 cache policy (reading R27; the paper's cache "follows HugeCTR", L1412-1414): every
    `epoch` steps the hot set is recomputed as the same per-table top-frequency rule (R10)
    over the `window` (default: epoch) steps just before the boundary t0 -- an LFU over a
    sliding window, decided from past traffic only.  Returns a copy carrying the schedule."""
    window = epoch if window is None else window
    sched = []
    for t0 in range(epoch, st.steps, epoch):
        lo = max(0, t0 - window)
        sched.append((t0, hot_set(st.cfg, st.ids[lo:t0], st.counts[lo:t0], window=t0 - lo)))
    return dataclasses.replace(st, hot_schedule=sched)


def stream_from_lists(cfg: WorkloadConfig, per_step: List[List[List[int]]],
                      x_value: float = 0.1) -> Stream:
    """Hand-written tiny stream (e.g. PAPER.md Fig. 6): per_step[s][g] = list of
    row ids (slots must be 1).  x = x_value * ones, y = 1."""
    assert cfg.slots == 1
    S, n = len(per_step), len(per_step[0])
    B = max(1, max(len(l) for st in per_step for l in st))
    cfg = dataclasses.replace(cfg, batch=B, world=n)
    ids = np.zeros((S, n, B), dtype=np.int64)
    counts = np.zeros((S, n), dtype=np.int32)
    for s in range(S):
        for g in range(n):
            l = per_step[s][g]
            ids[s, g, :len(l)] = l
            counts[s, g] = len(l)
    x = np.full((S, n, B, cfg.dim), x_value, dtype=np.float32)
    y = np.ones((S, n, B), dtype=np.float32)
    valid = (np.arange(B)[None, None, :] < counts[:, :, None])
    x[~valid] = 0
    y[~valid] = 0
    return Stream(cfg, ids, counts, x, y, np.zeros(0, dtype=np.int64))
