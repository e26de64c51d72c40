"""Thin ctypes binding of libfrugal.so (include/frugal.h).  Argument marshalling only:
every step of the hot path runs in the library's CUDA kernels.  There is no CPU
fallback: if the library is missing this module raises on import of the context.

Device buffers are torch CUDA tensors (PyTorch is plumbing: memory, streams,
process groups); host buffers are numpy arrays or pinned torch tensors.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(PKG, "libfrugal.so")

SGD, ADAGRAD = 0, 1
MODE_P2F, MODE_WRITE_THROUGH = 0, 1
F_RECORD, F_TIMERS, F_NO_HOST_STATE, F_A2A, F_PEER, F_DYNAMIC_CACHE, F_GPU_DRAIN, F_OWN_IDS = 1, 2, 4, 8, 16, 32, 64, 128
FLUSH_ALL = 0
PHASES = ["ingest", "schedule", "urgent", "gate", "gather", "expand", "model", "segred", "exchange",
          "optimizer", "side", "prefetch"]
_STATUS = {0: "FRUGAL_OK", -1: "FRUGAL_EINVAL", -2: "FRUGAL_ENOMEM", -3: "FRUGAL_ECUDA",
           -4: "FRUGAL_ESTATE", -5: "FRUGAL_ETIMEOUT", -6: "FRUGAL_ESHM"}


class FrugalError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


class Config(C.Structure):
    _fields_ = [("world", C.c_int32), ("rank", C.c_int32), ("device", C.c_int32), ("dim", C.c_int32),
                ("n_rows", C.c_int64), ("slots", C.c_int32), ("batch", C.c_int32), ("lookahead", C.c_int32),
                ("age_out", C.c_int32), ("opt", C.c_int32), ("lr", C.c_float), ("eps", C.c_float),
                ("init_accum", C.c_float), ("init_scale", C.c_float), ("init_seed", C.c_uint64),
                ("hot_ids", C.c_void_p), ("n_hot", C.c_int64), ("shm_name", C.c_char_p), ("mode", C.c_int32),
                ("flags", C.c_int32), ("host_order", C.c_void_p), ("n_order", C.c_int64),
                ("run_nonce", C.c_uint64)]


class ScheduleInfo(C.Structure):
    _fields_ = [("n_urgent", C.c_int64), ("n_deferred", C.c_int64), ("n_ageout", C.c_int64),
                ("gate_wait", C.c_int32)]


COUNTERS = ["positions", "unique", "gather_host", "gather_cache", "opt_hot", "opt_cold", "urgent_hot",
            "urgent_cold", "side_hot", "side_cold", "final_hot", "final_cold", "long_segments", "mail_out",
            "mail_in", "gather_pool", "gather_peer", "transition_hot", "transition_cold", "reserved19"]


class Stats(C.Structure):
    _fields_ = [("ms", C.c_double * 12), ("steps", C.c_int64), ("kernel_launches", C.c_int64),
                ("count", C.c_int64 * 20), ("flush_jobs", C.c_int64), ("flush_ms", C.c_double),
                ("flush_wait_ms", C.c_double), ("timer_steps", C.c_int64),
                ("host_wait_ms", C.c_double)]


_lib = None


def lib():
    """Load libfrugal.so; raises if it was not built (no fallback path exists)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: build it with `python -m paper_conf_asplos_xiezggl25_b200.build` "
                               "(or __graft_entry__.build()); there is no CPU fallback")
        L = C.CDLL(LIB_PATH)
        P, I64, I32 = C.c_void_p, C.c_int64, C.c_int32
        sig = {
            "frugal_init": [C.POINTER(Config), C.POINTER(P)],
            "frugal_prefetch": [P, I64, P, P, P],
            "frugal_step": [P, I64, P, P, P],
            "frugal_lookup": [P, I64, P, P],
            "frugal_backward_update": [P, I64, P, P],
            "frugal_flush": [P, I32, P],
            "frugal_destroy": [P],
            "frugal_dot_model": [P, I64, P, P, P, P, P, P],
            "frugal_transe_model": [P, I64, P, I32, C.c_float, P, P, P],
            "frugal_get_dedup": [P, I64, P, P, C.POINTER(I64)],
            "frugal_get_schedule": [P, C.POINTER(ScheduleInfo), P, P, P, P],
            "frugal_get_final_flush": [P, P, C.POINTER(I64)],
            "frugal_get_transition": [P, P, C.POINTER(I64)],
            "frugal_set_hot": [P, I64, P, I64],
            "frugal_read_rows": [P, P, I64, P, P],
            "frugal_read_host": [P, P, I64, P, P],
            "frugal_get_stats": [P, C.POINTER(Stats)],
            "frugal_get_timeline": [P, P, P, P, I64, C.POINTER(I64)],
            "frugal_probe_host_reads": [P, I64, C.c_uint64, C.POINTER(C.c_double)],
            "frugal_join": [P, P],
            "frugal_probe_fp64": [I32, C.POINTER(C.c_double)],
            "frugal_a2a_requests": [P, I64, P, P, P],
            "frugal_a2a_serve": [P, I64, P, I64, P, P],
            "frugal_a2a_lookup": [P, I64, P, P, P],
            "frugal_a2a_pack": [P, I64, P, P, P],
            "frugal_a2a_update": [P, I64, P, P, P],
        }
        for name, args in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = C.c_int
        L.frugal_last_error.restype = C.c_char_p
        L.frugal_last_error.argtypes = []
        L.frugal_owned_rows.restype = I64
        L.frugal_owned_rows.argtypes = [P]
        L.frugal_hot_slots.restype = I64
        L.frugal_hot_slots.argtypes = [P]
        _lib = L
    return _lib


EXPORTED = ["frugal_init", "frugal_prefetch", "frugal_step", "frugal_lookup", "frugal_backward_update",
            "frugal_flush", "frugal_destroy", "frugal_last_error", "frugal_dot_model", "frugal_transe_model",
            "frugal_get_dedup",
            "frugal_get_schedule", "frugal_get_final_flush", "frugal_read_rows", "frugal_read_host",
            "frugal_get_stats", "frugal_get_timeline", "frugal_owned_rows", "frugal_hot_slots",
            "frugal_a2a_requests", "frugal_a2a_serve", "frugal_a2a_lookup", "frugal_a2a_pack", "frugal_a2a_update",
            "frugal_probe_host_reads", "frugal_set_hot", "frugal_get_transition", "frugal_join",
            "frugal_probe_fp64"]


def _check(status):
    if status != 0:
        raise FrugalError(status, lib().frugal_last_error().decode())


def _ptr(x):
    """Pointer of a torch tensor / numpy array / int (None -> NULL)."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    return x.ctypes.data


_raw_stream = None


def _stream(stream):
    """cudaStream_t of `stream`; None = torch's current stream of the current device (read
    through torch's raw-stream accessor: no Python Stream object per call)."""
    global _raw_stream
    if stream is None:
        if _raw_stream is None:
            import torch
            try:
                get, dev = torch._C._cuda_getCurrentRawStream, torch._C._cuda_getDevice
                get(dev())
                _raw_stream = lambda: get(dev())
            except Exception:  # older torch: the public (slower) path
                _raw_stream = lambda: torch.cuda.current_stream().cuda_stream
        return _raw_stream()
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


class Frugal:
    """One rank's context (frugal_ctx).  Names follow frugal.h."""

    def __init__(self, *, world, rank, device, dim, n_rows, slots, batch, lookahead=10, age_out=10,
                 opt="adagrad", lr=0.05, eps=1e-10, init_accum=0.0, init_scale=0.05, init_seed=3, hot_ids=None,
                 shm_name=None, mode=MODE_P2F, flags=0, host_order=None, run_nonce=0):
        self.world, self.rank, self.dim, self.slots, self.batch = world, rank, dim, slots, batch
        self.flags = flags
        self.lookahead = lookahead
        hot = np.ascontiguousarray(np.zeros(0, np.int64) if hot_ids is None else hot_ids, dtype=np.int64)
        self._hot = hot
        self._shm = shm_name.encode() if shm_name else None
        order = np.ascontiguousarray(np.zeros(0, np.int64) if host_order is None else host_order, dtype=np.int64)
        self._order = order
        c = Config(world=world, rank=rank, device=device, dim=dim, n_rows=n_rows, slots=slots, batch=batch,
                   lookahead=lookahead, age_out=age_out, opt=ADAGRAD if opt == "adagrad" else SGD, lr=lr, eps=eps,
                   init_accum=init_accum, init_scale=init_scale, init_seed=init_seed,
                   hot_ids=hot.ctypes.data if hot.size else None, n_hot=hot.size, shm_name=self._shm, mode=mode,
                   flags=flags, host_order=order.ctypes.data if order.size else None, n_order=order.size,
                   run_nonce=run_nonce)
        self._cfg = c
        h = C.c_void_p()
        _check(lib().frugal_init(C.byref(c), C.byref(h)))
        self.h = h

    @classmethod
    def from_workload(cls, wcfg, *, world=None, rank=0, device=0, hot_ids=None, **kw):
        return cls(world=wcfg.world if world is None else world, rank=rank, device=device, dim=wcfg.dim,
                   n_rows=wcfg.n_rows, slots=wcfg.slots, batch=wcfg.batch, lookahead=wcfg.lookahead,
                   age_out=wcfg.age_out, opt=wcfg.opt, lr=wcfg.lr, eps=wcfg.eps, init_accum=wcfg.init_accum,
                   init_scale=wcfg.init_scale, init_seed=wcfg.seed_init, hot_ids=hot_ids, **kw)

    def close(self):
        if getattr(self, "h", None):
            lib().frugal_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ---- the hot path ---------------------------------------------------------------
    def prefetch(self, t, ids_all, counts, stream=None):
        counts = np.ascontiguousarray(counts, dtype=np.int32)
        _check(lib().frugal_prefetch(self.h, t, _ptr(ids_all), counts.ctypes.data, _stream(stream)))

    def step(self, s, ids_next_all=None, counts_next=None, stream=None):
        cn = None if counts_next is None else np.ascontiguousarray(counts_next, dtype=np.int32)
        _check(lib().frugal_step(self.h, s, _ptr(ids_next_all), None if cn is None else cn.ctypes.data,
                                 _stream(stream)))

    def lookup(self, s, out, stream=None):
        _check(lib().frugal_lookup(self.h, s, _ptr(out), _stream(stream)))

    def dot_model(self, s, emb, x, y, grad, loss, stream=None):
        _check(lib().frugal_dot_model(self.h, s, _ptr(emb), _ptr(x), _ptr(y), _ptr(grad), _ptr(loss),
                                      _stream(stream)))

    def transe_model(self, s, emb, chunk, gamma, grad, loss, stream=None):
        _check(lib().frugal_transe_model(self.h, s, _ptr(emb), chunk, gamma, _ptr(grad), _ptr(loss),
                                         _stream(stream)))

    def backward_update(self, s, grad, stream=None):
        _check(lib().frugal_backward_update(self.h, s, _ptr(grad), _stream(stream)))

    def flush(self, what=FLUSH_ALL, stream=None):
        _check(lib().frugal_flush(self.h, what, _stream(stream)))

    # ---- comparison path (FRUGAL_F_A2A) -------------------------------------------------
    def a2a_requests(self, s, ids_out, stream=None):
        """Fills ids_out (int32 device, >= n_uniq) grouped by owner; returns counts per owner."""
        counts = np.zeros(self.world, np.int64)
        _check(lib().frugal_a2a_requests(self.h, s, _ptr(ids_out), counts.ctypes.data, _stream(stream)))
        return counts

    def a2a_serve(self, s, ids_in, n_in, rows_out, stream=None):
        _check(lib().frugal_a2a_serve(self.h, s, _ptr(ids_in), n_in, _ptr(rows_out), _stream(stream)))

    def a2a_lookup(self, s, rows_in, out, stream=None):
        _check(lib().frugal_a2a_lookup(self.h, s, _ptr(rows_in), _ptr(out), _stream(stream)))

    def a2a_pack(self, s, grad, partials_out, stream=None):
        _check(lib().frugal_a2a_pack(self.h, s, _ptr(grad), _ptr(partials_out), _stream(stream)))

    def a2a_update(self, s, partials_in, recv_counts, stream=None):
        rc = np.ascontiguousarray(recv_counts, dtype=np.int64)
        _check(lib().frugal_a2a_update(self.h, s, _ptr(partials_in), rc.ctypes.data, _stream(stream)))

    # ---- introspection ---------------------------------------------------------------
    def get_dedup(self, t):
        n = C.c_int64()
        _check(lib().frugal_get_dedup(self.h, t, None, None, C.byref(n)))
        uq = np.empty(n.value, np.int64)
        inv = np.empty(self.batch * self.slots, np.int32)
        _check(lib().frugal_get_dedup(self.h, t, uq.ctypes.data, inv.ctypes.data, C.byref(n)))
        return uq, inv

    def get_schedule(self):
        info = ScheduleInfo()
        _check(lib().frugal_get_schedule(self.h, C.byref(info), None, None, None, None))
        u = np.empty(info.n_urgent, np.int64)
        dfr = np.empty(info.n_deferred, np.int64)
        dp = np.empty(info.n_deferred, np.int32)
        a = np.empty(info.n_ageout, np.int64)
        _check(lib().frugal_get_schedule(self.h, C.byref(info), u.ctypes.data, dfr.ctypes.data, dp.ctypes.data,
                                         a.ctypes.data))
        return dict(urgent=u, deferred=dfr, deferred_p=dp, ageout=a, gate_wait=bool(info.gate_wait))

    def set_hot(self, t0, hot_ids):
        """N3: the hot set from step t0 on (before step(t0 - L) / prefetch(t0))."""
        h = np.ascontiguousarray(hot_ids, dtype=np.int64)
        _check(lib().frugal_set_hot(self.h, int(t0), h.ctypes.data, len(h)))

    def get_transition(self):
        n = C.c_int64()
        _check(lib().frugal_get_transition(self.h, None, C.byref(n)))
        out = np.empty(n.value, np.int64)
        _check(lib().frugal_get_transition(self.h, out.ctypes.data, C.byref(n)))
        return out

    def get_final_flush(self):
        n = C.c_int64()
        _check(lib().frugal_get_final_flush(self.h, None, C.byref(n)))
        out = np.empty(n.value, np.int64)
        _check(lib().frugal_get_final_flush(self.h, out.ctypes.data, C.byref(n)))
        return out

    def read_rows(self, ids):
        ids = np.ascontiguousarray(ids, dtype=np.int64)
        w = np.empty((len(ids), self.dim), np.float32)
        G = np.empty((len(ids), self.dim), np.float32)
        _check(lib().frugal_read_rows(self.h, ids.ctypes.data, len(ids), w.ctypes.data, G.ctypes.data))
        return w, G

    def read_host(self, ids):
        ids = np.ascontiguousarray(ids, dtype=np.int64)
        w = np.empty((len(ids), self.dim), np.float32)
        G = np.empty((len(ids), self.dim), np.float32)
        _check(lib().frugal_read_host(self.h, ids.ctypes.data, len(ids), w.ctypes.data, G.ctypes.data))
        return w, G

    def get_stats(self):
        s = Stats()
        _check(lib().frugal_get_stats(self.h, C.byref(s)))
        return dict(ms={p: s.ms[i] for i, p in enumerate(PHASES)}, steps=s.steps,
                    kernel_launches=s.kernel_launches, count={n: s.count[i] for i, n in enumerate(COUNTERS)},
                    flush_jobs=s.flush_jobs, flush_ms=s.flush_ms, flush_wait_ms=s.flush_wait_ms,
                    timer_steps=s.timer_steps, host_wait_ms=s.host_wait_ms)

    def get_timeline(self, cap=4096):
        """[(phase name, start ms, end ms)] of the last `cap` recorded phases (all streams)."""
        ph = np.empty(cap, np.int32)
        t0 = np.empty(cap, np.float64)
        t1 = np.empty(cap, np.float64)
        n = C.c_int64()
        _check(lib().frugal_get_timeline(self.h, ph.ctypes.data, t0.ctypes.data, t1.ctypes.data, cap, C.byref(n)))
        return [(PHASES[ph[i]], float(t0[i]), float(t1[i])) for i in range(n.value)]

    def probe_host_reads(self, n, seed=12345):
        """ms to read n random host-table rows with the gather's pattern (calibration)."""
        ms = C.c_double()
        _check(lib().frugal_probe_host_reads(self.h, n, seed, C.byref(ms)))
        return ms.value

    def join(self, stream=None):
        """`stream` waits for all work enqueued on the library's own streams (timing)."""
        _check(lib().frugal_join(self.h, _stream(stream)))

    @property
    def owned_rows(self):
        return lib().frugal_owned_rows(self.h)

    @property
    def hot_slots(self):
        return lib().frugal_hot_slots(self.h)


def probe_fp64(device=0):
    """Separately rounded fp64 add/mul instructions per second of the device (calibration)."""
    r = C.c_double()
    _check(lib().frugal_probe_fp64(device, C.byref(r)))
    return r.value
