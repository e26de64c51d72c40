"""ctypes wrapper of the CPU oracle (oracle/frugal_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and the
cpu_baseline / --impl reference legs of bench.py.  The product path never
imports this module.  See frugal_oracle.c's header for what it computes and the
PAPER.md passages each part follows.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "frugal_oracle.c")
LIB = os.path.join(HERE, "liboracle.so")
# tools/oracle_mutants.py points this at a deliberately broken build (mutation testing of the pins)
LIB_OVERRIDE = os.environ.get("FRUGAL_ORACLE_LIB")

INF = 2**31 - 1
L_URGENT, L_DEFERRED, L_DEFERRED_P, L_AGEOUT, L_FINAL, L_UPDATED, L_INF, L_EXEMPT, L_TRANSITION = range(9)
CLEAN, UPDATED, INFP, EXEMPT = range(4)
MODELS = {"dot": 0, "const": 1, "l2": 2, "transe": 3}
OPTS = {"sgd": 0, "adagrad": 1}


class _Cfg(C.Structure):
    _fields_ = [("world", C.c_int32), ("dim", C.c_int32), ("slots", C.c_int32), ("batch", C.c_int32),
                ("lookahead", C.c_int32), ("age_out", C.c_int32), ("opt", C.c_int32), ("model", C.c_int32),
                ("n_rows", C.c_int64), ("lr", C.c_float), ("eps", C.c_float), ("init_accum", C.c_float),
                ("init_scale", C.c_float), ("init_seed", C.c_uint64), ("write_through", C.c_int32),
                ("skip_urgent_step", C.c_int32), ("gamma", C.c_float), ("neg_chunk", C.c_int32)]


def build(force: bool = False) -> str:
    """Compile the oracle (plain C, -O2, no FMA contraction, no fast-math)."""
    if LIB_OVERRIDE:
        return LIB_OVERRIDE
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math",
                               "-fPIC", "-shared", "-o", LIB, SRC, "-lm"])
    return LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        P, I64, I32 = C.c_void_p, C.c_int64, C.c_int32
        _lib.oracle_new.restype = P
        _lib.oracle_new.argtypes = [C.POINTER(_Cfg), P, I64]
        _lib.oracle_free.argtypes = [P]
        _lib.oracle_set_stream.argtypes = [P, I64, P, P, P, P]
        _lib.oracle_step.restype = I64
        _lib.oracle_step.argtypes = [P]
        _lib.oracle_final_flush.restype = I64
        _lib.oracle_final_flush.argtypes = [P]
        _lib.oracle_get_list.restype = I64
        _lib.oracle_get_list.argtypes = [P, C.c_int, P, I64]
        _lib.oracle_gate_wait.argtypes = [P]
        _lib.oracle_loss.restype = C.c_double
        _lib.oracle_loss.argtypes = [P, I64]
        _lib.oracle_violations.restype = I64
        _lib.oracle_violations.argtypes = [P]
        _lib.oracle_n_rows_touched.restype = I64
        _lib.oracle_n_rows_touched.argtypes = [P]
        _lib.oracle_dedup.restype = I64
        _lib.oracle_dedup.argtypes = [P, I64, I32, P, P]
        _lib.oracle_next_access.restype = I32
        _lib.oracle_next_access.argtypes = [P, I64, I64]
        _lib.oracle_needs_host.restype = I32
        _lib.oracle_needs_host.argtypes = [P, I64, I64]
        _lib.oracle_row_state.restype = I32
        _lib.oracle_row_state.argtypes = [P, I64]
        _lib.oracle_read_rows.argtypes = [P, P, I64, P, P]
        _lib.oracle_host_rows.argtypes = [P, P, I64, P, P]
        _lib.oracle_get_grad.argtypes = [P, I32, P]
        _lib.oracle_get_partial.restype = I64
        _lib.oracle_get_partial.argtypes = [P, I32, P, P]
        _lib.oracle_set_hot.restype = C.c_int
        _lib.oracle_set_hot.argtypes = [P, I64, P, I64]
        _lib.oracle_init_value.restype = C.c_float
        _lib.oracle_init_value.argtypes = [P, I64, I32]
    return _lib


def _p(a):
    return a.ctypes.data_as(C.c_void_p)


class Oracle:
    """Single-threaded synchronous trainer + brute-force P2F schedule."""

    def __init__(self, stream, model=None, opt=None, lookahead=None, age_out=None, lr=None,
                 write_through=False, skip_urgent_step=-1, hot=None):
        cfg = stream.cfg
        self.stream = stream
        self.world = stream.ids.shape[1]
        self.dim = cfg.dim
        self.slots = cfg.slots
        self.batch = stream.ids.shape[2] // cfg.slots
        c = _Cfg()
        c.world, c.dim, c.slots, c.batch = self.world, cfg.dim, cfg.slots, self.batch
        c.lookahead = cfg.lookahead if lookahead is None else lookahead
        c.age_out = cfg.age_out if age_out is None else age_out
        c.opt = OPTS[cfg.opt if opt is None else opt]
        c.model = MODELS[cfg.model if model is None else model]
        c.gamma, c.neg_chunk = cfg.gamma, cfg.neg_chunk
        c.n_rows = cfg.n_rows
        c.lr = cfg.lr if lr is None else lr
        c.eps, c.init_accum, c.init_scale = cfg.eps, cfg.init_accum, cfg.init_scale
        c.init_seed = cfg.seed_init
        c.write_through = int(write_through)
        c.skip_urgent_step = skip_urgent_step
        self.cfg = c
        hot = stream.hot if hot is None else hot
        self._hot = np.ascontiguousarray(hot, dtype=np.int64)
        self._keep = [np.ascontiguousarray(stream.ids, dtype=np.int64),
                      np.ascontiguousarray(stream.counts, dtype=np.int32),
                      np.ascontiguousarray(stream.x, dtype=np.float32),
                      np.ascontiguousarray(stream.y, dtype=np.float32)]
        L = lib()
        self.h = L.oracle_new(C.byref(c), _p(self._hot), len(self._hot))
        L.oracle_set_stream(self.h, stream.ids.shape[0], *[_p(a) for a in self._keep])
        for t0, ids in getattr(stream, "hot_schedule", None) or []:
            self.set_hot(t0, ids)

    def set_hot(self, t0, ids):
        """N3: the hot set from step t0 on (reading R27)."""
        a = np.ascontiguousarray(ids, dtype=np.int64)
        if lib().oracle_set_hot(self.h, int(t0), _p(a), len(a)) != 0:
            raise ValueError(f"oracle_set_hot({t0}): epochs must start after the previous one")

    def __del__(self):
        if getattr(self, "h", None):
            lib().oracle_free(self.h)
            self.h = None

    def step(self) -> int:
        return lib().oracle_step(self.h)

    def run(self, steps=None):
        n = self.stream.steps if steps is None else steps
        for _ in range(n):
            if self.step() < 0:
                break

    def final_flush(self) -> np.ndarray:
        lib().oracle_final_flush(self.h)
        return self.get_list(L_FINAL)

    def get_list(self, which) -> np.ndarray:
        n = lib().oracle_get_list(self.h, which, None, 0)
        out = np.empty(n, dtype=np.int64)
        lib().oracle_get_list(self.h, which, _p(out), n)
        return out

    def schedule(self):
        """Artefacts of the last step(): urgent, deferred (rows, deadlines), age-out, gate wait."""
        return dict(urgent=self.get_list(L_URGENT), deferred=self.get_list(L_DEFERRED),
                    deferred_p=self.get_list(L_DEFERRED_P), ageout=self.get_list(L_AGEOUT),
                    inf=self.get_list(L_INF), exempt=self.get_list(L_EXEMPT),
                    updated=self.get_list(L_UPDATED), transition=self.get_list(L_TRANSITION),
                    gate_wait=bool(lib().oracle_gate_wait(self.h)))

    def loss(self, s) -> float:
        return lib().oracle_loss(self.h, s)

    @property
    def violations(self) -> int:
        return lib().oracle_violations(self.h)

    def dedup(self, s, g):
        m = int(self.stream.counts[s, g]) * self.slots
        uq = np.empty(max(m, 1), dtype=np.int64)
        inv = np.empty(max(m, 1), dtype=np.int32)
        n = lib().oracle_dedup(self.h, s, g, _p(uq), _p(inv))
        return uq[:n].copy(), inv[:m].copy()

    def next_access(self, k, u) -> int:
        return lib().oracle_next_access(self.h, k, u)

    def needs_host(self, k, t) -> bool:
        return bool(lib().oracle_needs_host(self.h, k, t))

    def row_state(self, k) -> int:
        return lib().oracle_row_state(self.h, k)

    def read_rows(self, ks):
        ks = np.ascontiguousarray(ks, dtype=np.int64)
        w = np.empty((len(ks), self.dim), dtype=np.float32)
        G = np.empty((len(ks), self.dim), dtype=np.float32)
        lib().oracle_read_rows(self.h, _p(ks), len(ks), _p(w), _p(G))
        return w, G

    def host_rows(self, ks):
        ks = np.ascontiguousarray(ks, dtype=np.int64)
        w = np.empty((len(ks), self.dim), dtype=np.float32)
        G = np.empty((len(ks), self.dim), dtype=np.float32)
        lib().oracle_host_rows(self.h, _p(ks), len(ks), _p(w), _p(G))
        return w, G

    def grad(self, g):
        out = np.empty((self.batch * self.slots, self.dim), dtype=np.float32)
        lib().oracle_get_grad(self.h, g, _p(out))
        return out

    def partial(self, g):
        n = lib().oracle_get_partial(self.h, g, None, None)
        k = np.empty(n, dtype=np.int64)
        P = np.empty((n, self.dim), dtype=np.float32)
        lib().oracle_get_partial(self.h, g, _p(k), _p(P))
        return k, P

    def init_value(self, k, j) -> float:
        return lib().oracle_init_value(self.h, k, j)

    @property
    def n_touched(self) -> int:
        return lib().oracle_n_rows_touched(self.h)
