"""Training-loop harness around the C ABI (used by tests, bench.py and smoke()).

It only sequences the public calls of include/frugal.h for one rank:
prefetch(0..L-1), then per step: step(s) [enqueues step s+L] -> lookup(s) ->
dot_model(s) -> backward_update(s), and flush() at the end.  No arithmetic of the method
happens here.
"""
from __future__ import annotations

import numpy as np
import torch

from . import frugal as F


def make_context(st, rank=0, device=0, shm_name=None, flags=0, hot=None, mode=F.MODE_P2F, **over):
    cfg = st.cfg
    world = st.ids.shape[1]
    kw = dict(world=world, rank=rank, device=device, dim=cfg.dim, n_rows=cfg.n_rows, slots=cfg.slots,
              batch=st.ids.shape[2] // cfg.slots, lookahead=cfg.lookahead, age_out=cfg.age_out, opt=cfg.opt,
              lr=cfg.lr, eps=cfg.eps, init_accum=cfg.init_accum, init_scale=cfg.init_scale,
              init_seed=cfg.seed_init, hot_ids=st.hot if hot is None else hot, shm_name=shm_name, mode=mode,
              flags=flags)
    if getattr(st, "hot_schedule", None):
        kw["flags"] |= F.F_DYNAMIC_CACHE  # N3: the stream carries hot-set changes
    if getattr(st, "host_order", None) is not None:
        kw["host_order"] = st.host_order  # host-table layout (frugal_config.host_order)
    kw.update(over)
    return F.Frugal(**kw)


class Trainer:
    """Runs the stream on one rank.  Inputs are uploaded per step from host arrays."""

    def __init__(self, fr: F.Frugal, st, rank=0, device=0, fused_lookup=False, device_inputs=False,
                 host_inputs=False):
        self.fr, self.st, self.rank = fr, st, rank
        # fused lookup (REC glue only): lookup(s, None) + dot_model(s, None, ...) -- the
        # glue reads the gathered distinct rows through the inverse index, no expand
        self.fused = fused_lookup and st.cfg.model != "transe"
        self.dev = torch.device("cuda", device)
        # device_inputs: every step's ids (all ranks), x and y uploaded to HBM once, up front,
        # and passed as device pointers -- the bench's value leg; no host copy or host wait
        # inside the step loop, so the library's streams overlap exactly as in bench.py
        self.d_ids = self.d_x = self.d_y = None
        self.h_x = self.h_y = None
        if host_inputs:  # pinned host ids, x, y handed to the C ABI as host pointers (the e2e path)
            self.d_ids = torch.from_numpy(np.ascontiguousarray(st.ids)).pin_memory()
            self.h_x = torch.from_numpy(np.ascontiguousarray(st.x[:, rank])).pin_memory()
            self.h_y = torch.from_numpy(np.ascontiguousarray(st.y[:, rank])).pin_memory()
        if device_inputs:
            self.d_ids = torch.from_numpy(np.ascontiguousarray(st.ids)).to(self.dev)
            self.d_x = torch.from_numpy(np.ascontiguousarray(st.x[:, rank])).to(self.dev)
            self.d_y = torch.from_numpy(np.ascontiguousarray(st.y[:, rank])).to(self.dev)
        B, Fs, d = st.ids.shape[2] // st.cfg.slots, st.cfg.slots, st.cfg.dim
        self.emb = torch.empty(B * Fs, d, device=self.dev)
        self.grad = torch.empty_like(self.emb)
        self.loss = torch.zeros(st.steps, dtype=torch.float64, device=self.dev)
        self.s = 0
        # N3: hot set changes, handed to the library before the ingest of their t0
        self._hot = dict((int(t0), ids) for t0, ids in (getattr(st, "hot_schedule", None) or []))
        L = fr.lookahead
        for t in range(min(L, st.steps)):
            self._set_hot_before_ingest(t)
            fr.prefetch(t, self._ids(t), st.counts[t])

    def _ids(self, t):
        ids = self.st.ids[t] if self.d_ids is None else self.d_ids[t]
        # FRUGAL_F_OWN_IDS (ingest v2): the library gets this rank's ids only
        return ids[self.rank] if (self.fr.flags & F.F_OWN_IDS) and self.fr.world > 1 else ids

    def _set_hot_before_ingest(self, t):
        if t in self._hot:
            self.fr.set_hot(t, self._hot[t])

    def step(self, on_schedule=None):
        st, fr, s = self.st, self.fr, self.s
        t = s + fr.lookahead
        if t < st.steps:
            self._set_hot_before_ingest(t)
            fr.step(s, self._ids(t), st.counts[t])
        else:
            fr.step(s)
        if on_schedule:
            on_schedule(s)
        fr.lookup(s, None if self.fused else self.emb)
        if st.cfg.model == "transe":
            fr.transe_model(s, self.emb, st.cfg.neg_chunk, st.cfg.gamma, self.grad, self.loss[s:s + 1])
        elif self.d_x is not None:
            fr.dot_model(s, None if self.fused else self.emb, self.d_x[s], self.d_y[s], self.grad,
                         self.loss[s:s + 1])
        elif self.h_x is not None:
            fr.dot_model(s, None if self.fused else self.emb, self.h_x[s], self.h_y[s], self.grad,
                         self.loss[s:s + 1])
        else:
            x = torch.from_numpy(st.x[s, self.rank]).to(self.dev, non_blocking=False)
            y = torch.from_numpy(st.y[s, self.rank]).to(self.dev, non_blocking=False)
            fr.dot_model(s, None if self.fused else self.emb, x, y, self.grad, self.loss[s:s + 1])
        fr.backward_update(s, self.grad)
        self.s += 1

    def run(self, steps=None, on_schedule=None):
        n = self.st.steps if steps is None else steps
        while self.s < n:
            self.step(on_schedule)

    def losses(self):
        torch.cuda.synchronize(self.dev)
        return self.loss.cpu().numpy()


class A2ATrainer(Trainer):
    """The comparison path (Fig. 2b ❶-❺, L278-336): ids to their
    owners, rows back, partials to the owners, each by an all-to-all of the process group
    `group` (NCCL over NVLink on GPUs; gloo with host staging when `host_staging`, e.g.
    several ranks sharing one GPU in tests).  The context needs FRUGAL_F_A2A."""

    def __init__(self, fr, st, rank=0, device=0, dist=None, host_staging=False):
        super().__init__(fr, st, rank, device)
        self.dist = dist
        self.host = host_staging
        M, d = self.emb.shape
        self.ids_send = torch.empty(M, dtype=torch.int32, device=self.dev)
        self.part_send = torch.empty(M, d, device=self.dev)
        self.world = fr.world

    def _a2a(self, send, send_counts, recv_counts, inner):
        """all_to_all_single with per-rank row counts; inner = elements per row."""
        rc = [int(c) * inner for c in recv_counts]
        sc = [int(c) * inner for c in send_counts]
        src = send.reshape(-1)[:sum(sc)]
        if self.host:
            src = src.cpu()
        out = torch.empty(sum(rc), dtype=send.dtype, device=src.device)
        self.dist.all_to_all_single(out, src, rc, sc)
        return out.to(self.dev)

    def step(self, on_schedule=None):
        st, fr, s, D = self.st, self.fr, self.s, self.dist
        t = s + fr.lookahead
        if t < st.steps:
            self._set_hot_before_ingest(t)
            fr.step(s, self._ids(t), st.counts[t])
        else:
            fr.step(s)
        if on_schedule:
            on_schedule(s)
        d = self.emb.shape[1]
        send_counts = fr.a2a_requests(s, self.ids_send)                       # ❶ bucket by owner
        cdev = "cpu" if self.host else self.dev                               # NCCL: device tensors
        sc = torch.tensor(send_counts, dtype=torch.int64, device=cdev)
        rc = torch.empty_like(sc)
        D.all_to_all_single(rc, sc)                                            # counts
        recv_counts = rc.cpu().numpy()
        ids_in = self._a2a(self.ids_send, send_counts, recv_counts, 1)        # ❷ ids to owners
        rows_out = torch.empty(int(recv_counts.sum()), d, device=self.dev)
        fr.a2a_serve(s, ids_in, int(recv_counts.sum()), rows_out)             # ❸ owner queries
        torch.cuda.synchronize(self.dev)
        rows_in = self._a2a(rows_out, recv_counts, send_counts, d)            # ❹ rows back
        fr.a2a_lookup(s, rows_in, self.emb)                                    # ❺ reorder + expand
        if st.cfg.model == "transe":
            fr.transe_model(s, self.emb, st.cfg.neg_chunk, st.cfg.gamma, self.grad, self.loss[s:s + 1])
        else:
            x = torch.from_numpy(st.x[s, self.rank]).to(self.dev)
            y = torch.from_numpy(st.y[s, self.rank]).to(self.dev)
            fr.dot_model(s, self.emb, x, y, self.grad, self.loss[s:s + 1])
        fr.a2a_pack(s, self.grad, self.part_send)
        torch.cuda.synchronize(self.dev)
        part_in = self._a2a(self.part_send, send_counts, recv_counts, d)      # partials to owners
        fr.a2a_update(s, part_in, recv_counts)
        self.s += 1
