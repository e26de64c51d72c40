#!/usr/bin/env python
"""Benchmark of the Frugal training step on B200 (contract: one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...            (N > 1)

Workload: BASELINE.json configs[1], the Criteo-Kaggle-shaped DLRM embedding step
(26 tables, 33,762,577 rows, d = 32, fp32, Adagrad, Zipf alpha = 0.9, batch 8192 per
GPU, cache 5 %, L = 10), synthetic seeded ids.  A step is
one pass of the whole hot path: frugal_step (lookahead ingest + dedup + P2F bucketing
+ urgent flush + deferred drain on the side stream + gate) -> frugal_lookup (cache /
zero-copy host gather + expand) -> frugal_dot_model (glue) -> frugal_backward_update
(segment-reduce, mailbox exchange for N > 1, fused Adagrad).  Weak scaling: every rank
trains its own 8192-sample batch; all ranks share one host table in POSIX shm.

value  = samples/s with the step's inputs (ids of all ranks, x, y) already in HBM;
e2e    = samples/s through the same public calls with host (pinned) inputs copied
         in each step and the step's loss read back to the host;
roofline / per-phase rooflines use CUDA events recorded around every phase inside
the timed region (FRUGAL_F_TIMERS) and device row counters; cpu_baseline is the
oracle (oracle/, single thread) on a bounded sample of the same stream.
"""
import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "training samples/s at 1/2/4/8 B200; flush+gather GB/s vs HBM/host-link peak"
CONFIG_NAMES = {"tiny": "BASELINE.json configs[0]", "criteo_kaggle": "BASELINE.json configs[1]",
                "avazu": "BASELINE.json configs[2]", "freebase": "BASELINE.json configs[3]",
                "fb15k": "FB15k-shaped KG, Table 2", "criteo_tb": "BASELINE.json configs[4]"}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="criteo_kaggle")
    ap.add_argument("--alpha", type=float, default=0.9)
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--mode", default="p2f", choices=["p2f", "write_through"],
                    help="write_through = Frugal-Sync (every update flushed on the next step's critical path)")
    ap.add_argument("--exchange", default="host", choices=["host", "a2a"],
                    help="a2a = the comparison path: rows/partials by all-to-all over the process group "
                         "(NCCL/NVLink) instead of the host table and mailbox (N > 1)")
    ap.add_argument("--peer", action="store_true",
                    help="N4 NVLink-native variant: non-owned rows held in the owner's HBM are loaded "
                         "over peer memory instead of from the host table (N > 1)")
    ap.add_argument("--cache-refresh", type=int, default=0,
                    help="N3 dynamic cache: recompute the hot set every E steps (LFU over the previous E "
                         "steps, per-table top cache_ratio); 0 = static hot set")
    ap.add_argument("--host-layout", default="id", choices=["id", "freq"],
                    help="host-table layout: id order, or frequency order over the hot-set window "
                         "(frugal_config.host_order)")
    ap.add_argument("--no-fused-lookup", dest="fused_lookup", action="store_false",
                    help="expand the gathered rows to [B*F][d] in frugal_lookup and hand them to the glue; "
                         "default: the REC glue reads the gathered distinct rows through the inverse index "
                         "(frugal_lookup / frugal_dot_model with NULL emb, no expand; "
                         "profiles/r1_sweep32_fused_lookup.txt)")
    ap.add_argument("--drain", default="host", choices=["gpu", "host"],
                    help="deferred drain (a11): host (default) = packed by a kernel into a staging queue, copied "
                         "into the table by the library's flushing threads (PAPER.md L1055-1059); gpu = zero-copy "
                         "scatter kernel on the side stream (FRUGAL_F_GPU_DRAIN)")
    ap.add_argument("--ingest", default="v2", choices=["v1", "v2"],
                    help="N > 1: v2 (default) = each rank passes only its own ids, the ranks exchange distinct "
                         "ids through the host id mailbox (FRUGAL_F_OWN_IDS); v1 = every rank copies and scans "
                         "all ranks' ids")
    ap.add_argument("--host-gb", type=float, default=0.0,
                    help="criteo_tb (configs[4]): scale the Kaggle-profile tables to a host table of this many GB "
                         "(default: the full 8.8e8 rows if they fit in 45%% of this host's memory, else as many "
                         "rows as do)")
    ap.add_argument("--age-out", type=int, default=0,
                    help="override the config's age-out D (cold rows with no read in sight are flushed D "
                         "steps after their update; the owner's dirty-pool window is D+1 steps)")
    ap.add_argument("--timer-every", type=int, default=int(os.environ.get("FRUGAL_TIMER_EVERY", "1")),
                    help="phase timers (CUDA events around every phase) on every k-th step only: their "
                         "records cost the step a few %%; per-phase times are averages over the timed steps")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend for barriers / the max-over-ranks timing only")
    return ap.parse_args()


kSMs = 148


def source_sha():
    """Hash of the CUDA sources and the ABI header: ties a committed ncu capture to the code it measured."""
    import hashlib
    h = hashlib.sha256()
    csrc = os.path.join(ROOT, "paper_conf_asplos_xiezggl25_b200", "csrc")
    for f in sorted(os.listdir(csrc)):
        if f.endswith((".cu", ".cuh")):
            h.update(open(os.path.join(csrc, f), "rb").read())
    h.update(open(os.path.join(ROOT, "include", "frugal.h"), "rb").read())
    return h.hexdigest()[:12]


def dist_max(x, world, dist=None, device="cpu"):
    """Max of a per-rank float over all ranks (the contract's max-over-ranks timing)."""
    if world == 1:
        return x
    import torch
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def rank_device(local_rank):
    """One GPU per rank; FRUGAL_BENCH_SAME_DEVICE=1 puts every rank on cuda:0 (testing the
    multi-rank protocol on a one-GPU box)."""
    return 0 if os.environ.get("FRUGAL_BENCH_SAME_DEVICE") == "1" else local_rank


# ------------------------------------------------------------------------------ clocks
class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, dev):
        self.dev, self.rows, self.p = dev, [], None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.dev), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.p = None

    def _read(self):
        for line in self.p.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) == 6:
                self.rows.append(parts)

    def stop(self):
        if not self.p:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.p.terminate()
        self.p.wait()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[2 + i].lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


# ------------------------------------------------------------------------------ peaks
def host_link_peaks(torch, dev):
    """Pinned-copy peaks (1 GPU): H2D, D2H (256 MiB, best of 5, CUDA events)."""
    n = 256 << 20
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(n, dtype=torch.uint8, device=dev)
    out = {}
    for name, fn in [("h2d", lambda: d.copy_(h, non_blocking=True)), ("d2h", lambda: h.copy_(d, non_blocking=True))]:
        fn()
        torch.cuda.synchronize()
        best = 1e9
        for _ in range(5):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            b.synchronize()
            best = min(best, a.elapsed_time(b))
        out[name] = n / best / 1e6
    del h, d
    return out


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def gen_bench_stream(W, cfg, steps, layout="id"):
    """The seeded stream, minus the hot-set window: the static hot set is computed from the
    first HOT_WINDOW generated steps (reading R10), and the bench then trains on the steps
    AFTER them -- the cache is warmed from past traffic, never from the batches it times
    (timing those would credit the cache with a perfect forecast of its own steps)."""
    import dataclasses
    full = W.gen_stream(cfg, HOT_WINDOW + steps)
    # host-table layout from the same past window (frequency order)
    order = W.host_order(cfg, full.ids[:HOT_WINDOW], full.counts[:HOT_WINDOW]) if layout == "freq" else None
    return dataclasses.replace(full, ids=full.ids[HOT_WINDOW:], counts=full.counts[HOT_WINDOW:],
                               x=full.x[HOT_WINDOW:], y=full.y[HOT_WINDOW:], host_order=order)


HOT_WINDOW = 50


# ------------------------------------------------------------------------------ cpu baseline
def cpu_baseline(cfg, st, seconds):
    """The oracle as it stands (single thread) on the first steps of the same stream."""
    from oracle.oracle import Oracle
    o = Oracle(st)
    t0 = time.perf_counter()
    n = 0
    while n < st.steps and time.perf_counter() - t0 < seconds:
        o.step()
        n += 1
    dt = time.perf_counter() - t0
    B = st.ids.shape[2] // cfg.slots
    return {"value": n * B * st.ids.shape[1] / dt, "unit": "samples/s", "cores": 1, "kind": "oracle",
            "sample": f"first {n} steps of the {cfg.name} stream (world {st.ids.shape[1]}, batch {B}), "
                      f"{dt:.1f} s of single-thread C oracle incl. brute-force P2F schedule"}


# ------------------------------------------------------------------------------ reference arm
def run_reference(args, rank, world):
    if rank != 0:
        return
    from paper_conf_asplos_xiezggl25_b200 import workload as W
    cfg = W.config(args.config, world=1, alpha=args.alpha, **({"age_out": args.age_out} if args.age_out > 0 else {}))
    steps = args.warmup + args.steps
    # bounded sample: each "step" is one oracle step; cap the run to a few minutes
    per_step_budget = 60
    st = gen_bench_stream(W, cfg, min(steps, per_step_budget) + cfg.lookahead)
    from oracle.oracle import Oracle
    o = Oracle(st)
    for _ in range(min(args.warmup, 3)):
        o.step()
    K = min(args.steps, per_step_budget - min(args.warmup, 3))
    t0 = time.perf_counter()
    for _ in range(K):
        o.step()
    dt = time.perf_counter() - t0
    v = K * cfg.batch / dt
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "samples/s", "n_gpus": 1, "steps": K,
            "warmup": min(args.warmup, 3), "ms_per_step": dt / K * 1e3, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": cfg.name, "global_batch": cfg.batch, "tables": cfg.slots,
                       "rows": cfg.n_rows, "dim": cfg.dim, "alpha": cfg.alpha, "lookahead": cfg.lookahead,
                       "cache_ratio": cfg.cache_ratio, "opt": cfg.opt, "parallelism": "oracle, 1 CPU thread"},
            "e2e": {"value": v, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "cpu_baseline": {"value": v, "unit": "samples/s", "cores": 1, "kind": "oracle",
                             "sample": f"{K} oracle steps of the {cfg.name} stream after {min(args.warmup, 3)} "
                                       "warm-up steps (bounded sample)"}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------ our arm
def main():
    args = parse()
    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    if world != args.gpus and world == 1 and args.gpus > 1:
        sys.exit("--gpus N > 1 must be launched under torchrun with N processes")
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    import torch
    import torch.distributed as dist
    from paper_conf_asplos_xiezggl25_b200 import frugal as F
    from paper_conf_asplos_xiezggl25_b200 import workload as W
    from paper_conf_asplos_xiezggl25_b200.harness import make_context

    assert args.warmup >= 3, "timing rules: at least 3 warm-up steps"
    local = rank_device(local)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    coll_dev = dev if args.dist_backend == "nccl" else torch.device("cpu")
    if world > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")

    def barrier():
        if world > 1:
            dist.barrier()

    def max_over_ranks(x):
        return dist_max(x, world, dist, coll_dev)

    over = {}
    if args.config == "criteo_tb":  # configs[4]: 450 GB at full size -- rows scaled to the host's memory
        mem = os.sysconf("SC_PAGE_SIZE") * os.sysconf("SC_PHYS_PAGES")
        budget = args.host_gb * 1e9 if args.host_gb > 0 else 0.45 * mem
        over["rows_total"] = min(8.8e8, budget / (128 * 4))
    if args.age_out > 0:  # sensitivity of the lazy flush's holding time D (SURVEY Q9 default: the config's)
        over["age_out"] = args.age_out
    cfg = W.config(args.config, world=world, alpha=args.alpha, **over)
    K, Wm, L = args.steps, args.warmup, cfg.lookahead
    S = Wm + 2 * K + L + 2
    # at most SG distinct generated steps, cycled (step t reads generated step t % SG): the
    # generation stays bounded for any --steps, and SG id batches (>= 400 MB at configs[1])
    # still exceed the 126 MB L2
    SG = min(S, 256)
    t_gen = time.time()
    st = gen_bench_stream(W, cfg, SG, args.host_layout)  # every rank generates the same seeded stream of all ranks
    t_gen = time.time() - t_gen
    B, Fs, d = cfg.batch, cfg.slots, cfg.dim
    shm = f"/frugal_bench_{os.environ.get('MASTER_PORT', '0')}" if world > 1 else None
    host_bytes = cfg.n_rows * 4 * d * (2 if cfg.opt == "adagrad" else 1)
    no_host_state = host_bytes > 150e9  # configs[3]: w + G do not both fit in host RAM
    a2a = args.exchange == "a2a"
    if a2a and world == 1:
        sys.exit("--exchange a2a needs N > 1")
    nonce = 0
    if world > 1:  # one run id for the shared segment, drawn by rank 0 (frugal_config.run_nonce)
        t = torch.tensor([int.from_bytes(os.urandom(7), "little") | 1 if rank == 0 else 0], dtype=torch.int64,
                         device=coll_dev)
        dist.broadcast(t, 0)
        nonce = int(t.item())
    os.environ["FRUGAL_TIMER_EVERY"] = str(max(1, args.timer_every))  # read by frugal_init
    fr = make_context(st, rank=rank, device=local, shm_name=shm, run_nonce=nonce,
                      flags=F.F_TIMERS | (F.F_NO_HOST_STATE if no_host_state else 0) | (F.F_A2A if a2a else 0)
                      | (F.F_PEER if (args.peer and world > 1) else 0)
                      | (F.F_DYNAMIC_CACHE if args.cache_refresh > 0 else 0)
                      | (F.F_GPU_DRAIN if args.drain == "gpu" else 0)
                      | (F.F_OWN_IDS if (args.ingest == "v2" and world > 1) else 0),
                      mode=F.MODE_WRITE_THROUGH if args.mode == "write_through" else F.MODE_P2F)
    # N3: the hot set of every epoch start t0 (bench step numbering; step t reads generated
    # step t % SG), from the E bench steps before t0 -- inputs, computed before any timing,
    # pinned so that frugal_set_hot copies them asynchronously
    hot_at = {}
    E = args.cache_refresh
    if E > 0:
        if E <= L:
            sys.exit("--cache-refresh must exceed the lookahead")
        for t0 in range(E, S, E):
            win = np.stack([st.ids[t % SG] for t in range(t0 - E, t0)])
            cw = np.stack([st.counts[t % SG] for t in range(t0 - E, t0)])
            hot_at[t0] = torch.from_numpy(W.hot_set(cfg, win, cw, window=E)).pin_memory()

    def set_hot_before_ingest(t):
        if t in hot_at:
            fr.set_hot(t, hot_at[t].numpy())
    barrier()
    stream = torch.cuda.current_stream(dev)

    # inputs of the value leg resident in HBM
    ids_d = torch.from_numpy(st.ids).to(dev)                       # [S][world][M] int64
    x_d = torch.from_numpy(np.ascontiguousarray(st.x[:, rank])).to(dev)
    y_d = torch.from_numpy(np.ascontiguousarray(st.y[:, rank])).to(dev)
    emb = torch.empty(B * Fs, d, device=dev)
    grad = torch.empty_like(emb)
    loss = torch.zeros(S, dtype=torch.float64, device=dev)
    # pinned host copies for the e2e leg
    own = args.ingest == "v2" and world > 1  # FRUGAL_F_OWN_IDS: the library gets this rank's ids only
    ids_h = torch.from_numpy(np.ascontiguousarray(st.ids[:, rank] if own else st.ids)).pin_memory()
    if own:
        ids_d = ids_d[:, rank].contiguous()
    x_h = torch.from_numpy(np.ascontiguousarray(st.x[:, rank])).pin_memory()
    y_h = torch.from_numpy(np.ascontiguousarray(st.y[:, rank])).pin_memory()
    loss_h = torch.zeros(S, dtype=torch.float64).pin_memory()
    counts = st.counts

    for t in range(L):
        set_hot_before_ingest(t)
        fr.prefetch(t, ids_d[t % SG], counts[t % SG])

    kg = cfg.model == "transe"
    host_staging = args.dist_backend == "gloo"
    ids_send = torch.empty(B * Fs, dtype=torch.int32, device=dev)
    part_send = torch.empty(B * Fs, d, device=dev)

    def a2a_xchg(send, send_counts, recv_counts, inner):
        rc = [int(c) * inner for c in recv_counts]
        sc = [int(c) * inner for c in send_counts]
        src = send.reshape(-1)[:sum(sc)]
        if host_staging:
            src = src.cpu()
        out = torch.empty(sum(rc), dtype=send.dtype, device=src.device)
        dist.all_to_all_single(out, src, rc, sc)
        return out.to(dev, non_blocking=True)

    fused = args.fused_lookup and not kg and not a2a
    emb_arg = None if fused else emb

    def lookup(s):
        if not a2a:
            fr.lookup(s, emb_arg, stream=stream.cuda_stream)
            return
        sc = fr.a2a_requests(s, ids_send)
        sct = torch.tensor(sc, dtype=torch.int64, device=coll_dev)
        rct = torch.empty_like(sct)
        dist.all_to_all_single(rct, sct)
        rc = rct.cpu().numpy()
        ids_in = a2a_xchg(ids_send, sc, rc, 1)
        rows_out = torch.empty(int(rc.sum()), d, device=dev)
        fr.a2a_serve(s, ids_in, int(rc.sum()), rows_out)
        rows_in = a2a_xchg(rows_out, rc, sc, d)
        fr.a2a_lookup(s, rows_in, emb)
        lookup.counts = (sc, rc)

    def backward(s):
        if not a2a:
            fr.backward_update(s, grad, stream=stream.cuda_stream)
            return
        sc, rc = lookup.counts
        fr.a2a_pack(s, grad, part_send)
        part_in = a2a_xchg(part_send, sc, rc, d)
        fr.a2a_update(s, part_in, rc)

    # per-step views and counts made once: the step loop is a handful of C-ABI calls
    ids_v = [ids_d[t] for t in range(SG)]
    ids_hv = [ids_h[t] for t in range(SG)]
    x_v = [x_d[t] for t in range(SG)]
    y_v = [y_d[t] for t in range(SG)]
    loss_v = [loss[t:t + 1] for t in range(S)]
    cnt_v = [np.ascontiguousarray(counts[t], dtype=np.int32) for t in range(SG)]
    sh = stream.cuda_stream

    def step_dev(s):
        t = s + L
        set_hot_before_ingest(t)
        fr.step(s, ids_v[t % SG], cnt_v[t % SG], stream=sh)
        lookup(s)
        if kg:
            fr.transe_model(s, emb, cfg.neg_chunk, cfg.gamma, grad, loss_v[s], stream=sh)
        else:
            fr.dot_model(s, emb_arg, x_v[s % SG], y_v[s % SG], grad, loss_v[s], stream=sh)
        backward(s)

    x_hv = [x_h[t] for t in range(SG)]
    y_hv = [y_h[t] for t in range(SG)]
    loss_hv = [loss_h[t:t + 1] for t in range(S)]

    def step_e2e(s):
        # every input from pinned host memory through the C ABI: ids in frugal_step, x and y in
        # frugal_dot_model (copied by the library); the step's loss read back to the host
        t = s + L
        set_hot_before_ingest(t)
        fr.step(s, ids_hv[t % SG], cnt_v[t % SG], stream=sh)
        lookup(s)
        if kg:
            fr.transe_model(s, emb, cfg.neg_chunk, cfg.gamma, grad, loss_v[s], stream=sh)
        else:
            fr.dot_model(s, emb_arg, x_hv[s % SG], y_hv[s % SG], grad, loss_v[s], stream=sh)
        backward(s)
        loss_hv[s].copy_(loss_v[s], non_blocking=True)  # the step's result back to the host

    # ---- warm-up
    for s in range(Wm):
        step_dev(s)
    torch.cuda.synchronize()
    fr.get_stats()  # reset phase timers / read counters
    st0 = fr.get_stats()
    # ---- value leg (inputs in HBM)
    clocks = Clocks(local)
    clocks.start()
    barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for s in range(Wm, Wm + K):
        step_dev(s)
    fr.join(stream)  # the last steps' ingest (s+L) and side drain belong to the timed work
    e1.record(stream)
    torch.cuda.synchronize()
    barrier()
    ms = e0.elapsed_time(e1)
    clk = clocks.stop()
    st1 = fr.get_stats()
    ms_max = max_over_ranks(ms)
    value = world * B * K / (ms_max / 1e3)

    # ---- e2e leg (host inputs, loss read back)
    barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f0.record(stream)
    for s in range(Wm + K, Wm + 2 * K):
        step_e2e(s)
    fr.join(stream)
    f1.record(stream)
    torch.cuda.synchronize()
    wall = time.perf_counter() - t0
    barrier()
    e2e_ms = max_over_ranks(max(f0.elapsed_time(f1), wall * 1e3))
    e2e = world * B * K / (e2e_ms / 1e3)
    fr.get_stats()
    finite = bool(torch.isfinite(loss[Wm:Wm + 2 * K]).all().item())

    # ---- per-phase rooflines for this rank
    cnt = {k: st1["count"][k] - st0["count"][k] for k in st1["count"]}
    # ms per step (per launch of the phase), averaged over the steps the timers covered
    ph = {k: v / max(1, st1["timer_steps"]) for k, v in st1["ms"].items()}
    r = 4 * d
    adag = cfg.opt == "adagrad"
    peaks = measured_peaks()
    link = host_link_peaks(torch, dev)
    # random-row ceiling of this box: fresh pseudo-random rows of the host table, gather pattern
    nprobe = max(1, int(cnt["gather_host"] / K))
    probe = [fr.probe_host_reads(nprobe, seed=1000 + i) for i in range(3)]
    link["random_rows_h2d"] = nprobe * r / (min(probe) * 1e-3) / 1e9
    hbm_peak = peaks.get("hbm_gbs", 6650.0)

    def gbs(nbytes, ms_):
        return nbytes / (ms_ * 1e-3) / 1e9 if ms_ > 0 else None

    per = {}
    # Algorithmic bytes per unit, times the units the device counters saw.
    # a4 gather: r per unique row served from the host table (zero-copy, PCIe H2D) -- the miss path
    per["gather"] = dict(bound="host-link h2d", bytes=cnt["gather_host"] * r / K,
                         hbm_bytes=(cnt["gather_cache"] + cnt["gather_pool"] + cnt["unique"]) * r / K,
                         ms=ph["gather"], peak=link["h2d"])
    if ph.get("prefetch", 0.0) > 0.0:
        # early gather (world 1, FRUGAL_EARLY): every host row of step s+1 is read by the early
        # gather on the library's prefetch stream during step s (the lag rule); the main-stream
        # gather of s+1 reads only the rows updated at s (HBM: pool / cache)
        per["gather"].update(ms=ph["prefetch"], kernel="k_gather_uniq_r (early part: host rows, prefetch stream)",
                             main_stream_ms=ph["gather"])
    # a10 urgent flush (critical path) / a11 side drain: r per flushed row (w only, R8), D2H
    for nm, h, c_ in [("urgent", "urgent_hot", "urgent_cold"), ("side", "side_hot", "side_cold")]:
        per[nm] = dict(bound="host-link d2h", bytes=(cnt[h] + cnt[c_]) * r / K, ms=ph[nm], peak=link["d2h"])
    if ph["urgent"] == 0.0 and cnt["urgent_hot"] + cnt["urgent_cold"] > 0:
        # world 1: the urgent bucket is packed with the step's drain job (reading R7')
        per["side"]["bytes"] += (cnt["urgent_hot"] + cnt["urgent_cold"]) * r / K
        per["side"]["note"] = "drain pack incl. the urgent bucket (world 1); side ms include the wait for a free staging buffer"
        per["urgent"]["bytes"] = 0.0
    # a4 expand: out[i] = rows[inv[i]]: write r + read r + 4 B index per position
    per["expand"] = dict(bound="hbm", bytes=0.0 if fused else (cnt["positions"] * (2 * r + 4)) / K,
                         ms=ph["expand"], peak=hbm_peak)
    # a6 segment-reduce: read r + 4 B per position, write r + 4 B per unique row
    per["segred"] = dict(bound="hbm", bytes=(cnt["positions"] * (r + 4) + cnt["unique"] * (r + 4)) / K,
                         ms=ph["segred"], peak=hbm_peak)
    # a8 optimizer: per touched owned row: partial r, w r (cache / staged rows), G r+r, w out r,
    # + 28 B metadata; cold rows of other ranks' reads come over the link when N > 1
    touched = cnt["opt_hot"] + cnt["opt_cold"]
    per["optimizer"] = dict(bound="hbm", bytes=touched * (5 * r + 28) / K,
                            link_bytes=(cnt["opt_cold"] * r + cnt["mail_in"] * r) / K if world > 1 else 0.0,
                            ms=ph["optimizer"], peak=hbm_peak)
    if world == 1 and ph["optimizer"] == 0.0 and ph["segred"] > 0.0:
        # world 1: the optimizer is fused into the segment-reduce (one pass, no partials buffer):
        # per position r + 4 B (grad row, pos); per touched row w r, G r + r, w out r, 28 B metadata
        per["segred"] = dict(bound="hbm", kernel="k_update1 (a6 + a8 fused, one launch)",
                             bytes=(cnt["positions"] * (r + 4) + touched * (4 * r + 28)) / K,
                             ms=ph["segred"], peak=hbm_peak)
        per["optimizer"]["bytes"] = 0.0
    # a5 glue: read r per position (embeddings, register-cached), write r (grads), x per sample
    per["model"] = dict(bound="hbm", bytes=(cnt["positions"] * 2 * r + B * (r + 4)) / K, ms=ph["model"],
                        peak=hbm_peak)
    if kg:
        # a5 KG glue (TransE, R26): fp64 ALU-bound, not HBM.  Algorithmic ops per chunk of C
        # triples with C shared negatives: distances C*C*d*3 (sub, mul, add), the two gradient
        # reductions 2*C*C*d*3; positives d*4 per triple.  Every op is a separately rounded
        # DADD/DSUB/DMUL (no FMA), so the peak is the fp64 instruction rate, measured in this run
        # by frugal_probe_fp64 (all SMs, independent DADD/DMUL chains) next to its derivation
        # SMs x fp64 lanes per SM x clock.
        cnt_b = B  # triples per rank per step (full batches in the bench)
        C_ = cfg.neg_chunk
        nch, last = cnt_b // C_, cnt_b % C_
        pairs = nch * C_ * C_ + last * last
        flops = pairs * d * 9 + cnt_b * d * 4
        fp64_peak = F.probe_fp64(local) / 1e12
        per["model"] = dict(bound="alu", flops=flops, ms=ph["model"], peak_tflops=fp64_peak,
                            achieved_tflops=flops / (ph["model"] * 1e-3) / 1e12 if ph["model"] > 0 else None)
        per["model"]["frac"] = (per["model"]["achieved_tflops"] / fp64_peak) if per["model"]["achieved_tflops"] else None
    for k, v in per.items():
        if v.get("bound") == "alu":
            continue
        v["achieved_gbs"] = gbs(v["bytes"], v["ms"])
        v["frac"] = v["achieved_gbs"] / v["peak"] if v["achieved_gbs"] else None
    # phases on the caller's (main) stream; ingest, side drain and early gather run on library streams
    main_ms = {k: v for k, v in ph.items() if k not in ("side", "ingest", "prefetch")}
    dom = max(("gather", "urgent", "expand", "segred", "optimizer", "model"), key=lambda k: per[k]["ms"])
    top = max(main_ms, key=main_ms.get)
    D = per[dom]
    traffic, tnote, htraffic = None, None, None
    try:  # committed ncu --set full capture (tools/profile_round.sh -> tools/ncu_summary.py)
        cap = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json"))).get(cfg.name, {})
        prof = cap.get("kernels", {}).get(dom, {})
        if prof:
            if cap.get("source_sha") == source_sha():
                traffic = prof.get("traffic_bytes_per_launch")
                htraffic = prof.get("host_link_bytes_per_launch")
                tnote = (f"dram read+write per launch of {prof['kernel']}: mean of {prof['launches_profiled']} "
                         f"steady-state launches, ncu --set full of this config on this source "
                         f"(sha {cap['source_sha']}, {cap.get('file', 'profiles/')}); host_link_traffic = its "
                         f"sysmem sectors through L2")
            else:
                tnote = (f"null: the committed ncu capture of {cfg.name} (source sha {cap.get('source_sha')}) "
                         f"predates this source (sha {source_sha()})")
        else:
            tnote = f"null: no committed ncu capture of {dom} for {cfg.name}"
    except Exception as e:
        tnote = f"null: {e}"
    if D.get("bound") != "alu":
        roofline = {"bound": "hbm" if D["bound"] == "hbm" else "host-link", "kernel": D.get("kernel", dom),
                    "achieved": D["achieved_gbs"], "peak": D["peak"], "unit": "GB/s", "frac": D["frac"],
                    # a uniform-random probe over the whole table is a reference rate, not a
                    # ceiling -- the step's host rows follow the Zipf tail and beat it
                    "random_row_reference": link["random_rows_h2d"] if D["bound"] != "hbm" else None,
                    "ratio_to_random_row_reference": (D["achieved_gbs"] / link["random_rows_h2d"])
                    if D["bound"] != "hbm" and D["achieved_gbs"] else None,
                    "translation_note": ("on the B200 boxes of this round (KVM guests: GPU DMA through the host IOMMU) the gather is bound by translating random host "
                                         "addresses: the same gather from a 512 MB "
                                         "footprint reaches 0.55-0.57 of this peak (profiles/r2_sweep_translation.txt)")
                    if D["bound"] != "hbm" else None,
                    "traffic": traffic, "host_link_traffic": htraffic, "traffic_note": tnote,
                    "peak_source": ("measured pinned cudaMemcpy (256 MiB, best of 5) in this run; random 128-B rows "
                                    "measure 12-33 GB/s on this box (profiles/r1_zc_probe_*.txt), the step's exact host-row "
                                    "list replayed alone 25-27 GB/s (profiles/r1_exact_replay.txt)" if D["bound"] != "hbm"
                                    else "MEASURED_PEAKS.json hbm_gbs (burst)")}
    else:  # KG glue dominates: fp64 ALU roofline
        roofline = {"bound": "alu", "kernel": dom + " (k_transe_pos / _pairs_tiled / _grads_tiled)",
                    "achieved": D["achieved_tflops"], "peak": D["peak_tflops"], "unit": "TFLOP/s", "frac": D["frac"],
                    "traffic": None,
                    "peak_source": "fp64 add/mul instruction rate measured in this run by frugal_probe_fp64 "
                                   "(every op of the KG glue is one such instruction, DESIGN.md §7)",
                    "peak_derived": kSMs * 64 * (clk.get("sm_max_mhz") or 1965.0) * 1e6 / 1e12,
                    "peak_derived_note": "148 SMs x 64 fp64 lanes x max SM clock (1 op per lane per clock)"}
    launches = st1["kernel_launches"] - st0["kernel_launches"]
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(cfg, st, args.cpu_seconds)  # the oracle on the first steps of the same stream
    # ids (this rank's with ingest v2, all ranks' with v1), x, y, counts
    h2d = int((1 if own else world) * B * Fs * 8 + B * d * 4 + B * 4 + world * 4)
    line = {
        "metric": METRIC, "value": value, "unit": "samples/s", "n_gpus": world, "steps": K, "warmup": Wm,
        "ms_per_step": ms_max / K, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "f32", "data": "synthetic",
        "config": {"workload": f"{cfg.name} ({CONFIG_NAMES.get(cfg.name, '')})", "global_batch": world * B,
                   "batch_per_gpu": B, "tables": Fs, "rows": cfg.n_rows, "dim": d, "alpha": cfg.alpha,
                   "rows_note": ("the Kaggle profile scaled to %.3g rows (%.0f GB host table) to fit this host's "
                                 "memory; configs[4] is 8.8e8 rows / 450 GB" % (cfg.n_rows, cfg.n_rows * d * 4 / 1e9))
                   if cfg.name == "criteo_tb" and cfg.n_rows < 8.7e8 else None,
                   "lookahead": L, "age_out": cfg.age_out, "cache_ratio": cfg.cache_ratio, "opt": cfg.opt,
                   "flush_mode": args.mode,
                   "drain": "side-stream zero-copy scatter kernel" if args.drain == "gpu" else
                            "packed staging queue + library flushing threads (default)",
                   "exchange": "host table + mailbox (P2F)" if not a2a else
                   "all-to-all over the process group (comparison path)",
                   "peer_reads": bool(args.peer and world > 1),
                   "ingest": ("v2: own ids, distinct ids exchanged through the host id mailbox" if own else
                              "v1: every rank scans all ranks' ids") if world > 1 else "world 1",
                   "lookup": "fused into the glue (no expand)" if fused else "expanded [B*F][d]",
                   "parallelism": f"dp{world} (owner-sharded rows, shared pinned host table)",
                   "l2": "inputs larger than L2: host table %.1f GB, HBM cache %.0f MB, %d distinct id batches "
                         "(%.0f MB) cycled" % (cfg.n_rows * r * (1 if (no_host_state or not adag) else 2) / 1e9,
                                               len(st.hot) * r / 1e6, SG, st.ids.nbytes / 1e6),
                   "host_layout": ("frequency order over the %d generated steps before the bench's first step "
                                   "(frugal_config.host_order)" % HOT_WINDOW) if args.host_layout == "freq" else "id order",
                   "hot_set": "top cache_ratio of each table by frequency over the %d generated steps before "
                              "the bench's first step (never over timed steps)" % HOT_WINDOW,
                   "host_state": "w only (G HBM-resident, no host copy)" if no_host_state else "w (+G at final flush)",
                   "cache": ("dynamic (N3): hot set recomputed every %d steps, per-table top cache_ratio by "
                             "frequency over the previous %d steps" % (E, E)) if E > 0 else "static"},
        "e2e": {"value": e2e, "unit": "samples/s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": 8},
        "gpu_launches": int(launches),
        "roofline": roofline,
        "phases_ms_per_step": {k: round(v, 5) for k, v in ph.items()},
        "phase_timers": {"every": max(1, args.timer_every), "timed_steps": int(st1["timer_steps"])},
        "rooflines": {k: {kk: (round(vv, 4) if isinstance(vv, float) else vv) for kk, vv in v.items()}
                      for k, v in per.items()},
        "flush_gather_gbs": {"gather_host_h2d": per["gather"]["achieved_gbs"],
                             "flush_urgent_d2h": per["urgent"]["achieved_gbs"],
                             "flush_side_d2h": per["side"]["achieved_gbs"],
                             "host_link_peak": link, "hbm_peak": hbm_peak},
        "rows_per_step": {k: v / K for k, v in cnt.items()},
        "flushing_threads": {"jobs": st1.get("flush_jobs"), "copy_ms_per_job": (st1["flush_ms"] / st1["flush_jobs"])
                             if st1.get("flush_jobs") else None,
                             "wait_ms_per_job": (st1["flush_wait_ms"] / st1["flush_jobs"])
                             if st1.get("flush_jobs") else None},
        "top_main_stream_phase": top,
        "clocks": clk,
        "loss_finite": finite,
        "gen_s": round(t_gen, 1),
    }
    if cpu:
        line["cpu_baseline"] = cpu
    fr.close()
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
