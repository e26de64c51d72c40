"""world = 2 on ONE B200: two rank processes share device 0 and one POSIX-shm host
table; mailboxes, flags and gates go through host memory exactly as across GPUs.
Compared against the oracle run with world 2: per-rank schedule sets (each rank owns
k mod 2 == rank), final flush, host table (w, G) and the global loss."""
import multiprocessing as mp
import os
import traceback

import numpy as np
import pytest

from paper_conf_asplos_xiezggl25_b200 import workload as W

pytestmark = pytest.mark.gpu


def _rank_main(rank, st, shm, barrier, q, a2a=False, port=0, peer=False, fused=False, nonce=1):
    try:
        import torch
        from paper_conf_asplos_xiezggl25_b200 import frugal as F
        from paper_conf_asplos_xiezggl25_b200.harness import A2ATrainer, Trainer, make_context
        torch.cuda.set_device(0)
        fr = make_context(st, rank=rank, device=0, shm_name=shm, run_nonce=nonce,
                          flags=F.F_RECORD | (F.F_A2A if a2a else 0) | (F.F_PEER if peer else 0))
        barrier.wait()
        if a2a:
            import torch.distributed as dist
            os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
            dist.init_process_group("gloo", rank=rank, world_size=2)
            tr = A2ATrainer(fr, st, rank=rank, dist=dist, host_staging=True)
        else:
            tr = Trainer(fr, st, rank=rank, fused_lookup=fused)
        sched = []
        for s in range(st.steps):
            got = {}

            def cb(s_):
                got.update(fr.get_schedule())
                got["transition"] = fr.get_transition()
            tr.step(on_schedule=cb)
            sched.append(got)
        fr.flush()
        ff = fr.get_final_flush()
        losses = tr.losses()
        stats = fr.get_stats()["count"]
        barrier.wait()  # both ranks flushed: the host table is authoritative
        w = G = None
        if rank == 0:
            w, G = fr.read_host(np.arange(st.cfg.n_rows))
        barrier.wait()
        fr.close()
        q.put((rank, dict(sched=sched, ff=ff, losses=losses, w=w, G=G, stats=stats)))
    except Exception:
        q.put((rank, traceback.format_exc()))


def run_two_ranks(st, timeout=600, a2a=False, peer=False, fused=False):
    import socket
    ctx = mp.get_context("spawn")
    barrier = ctx.Barrier(2)
    q = ctx.Queue()
    shm = f"/frugal_test_{os.getpid()}"
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    nonce = int.from_bytes(os.urandom(8), "little") | 1
    ps = [ctx.Process(target=_rank_main, args=(r, st, shm, barrier, q, a2a, port, peer, fused, nonce))
          for r in range(2)]
    for p in ps:
        p.start()
    out = {}
    try:
        for _ in range(2):
            r, v = q.get(timeout=timeout)
            out[r] = v
    finally:
        for p in ps:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    for r, v in out.items():
        assert not isinstance(v, str), f"rank {r} failed:\n{v}"
    return out


@pytest.mark.parametrize("opt,a2a,peer,dyn,layout", [("adagrad", False, False, False, False),
                                                     ("sgd", False, False, False, False),
                                                     ("adagrad", True, False, False, False),
                                                     ("adagrad", False, True, False, False),
                                                     ("adagrad", False, False, True, False),
                                                     ("adagrad", False, False, False, True)])
def test_two_ranks_one_gpu_parity(opt, a2a, peer, dyn, layout):
    """a2a=True: the comparison path (§8(e)) -- ids, rows and partials move by all-to-all
    (gloo with host staging here; NCCL over NVLink on a multi-GPU box) instead of the host
    table and mailbox; every artefact and table must be identical.  peer=True: the N4
    variant -- non-owned rows the owner holds in HBM are loaded from the owner's device
    memory (CUDA IPC; NVLink on a multi-GPU box); every artefact and table identical.
    layout=True: both ranks share a host table laid out by a random partial host_order
    (frugal_config.host_order); every artefact and table identical."""
    from oracle.oracle import Oracle
    cfg = W.config("tiny", world=2, batch=64, lookahead=4, age_out=3, opt=opt,
                   lr=0.05 if opt == "adagrad" else 1.0)
    rng = np.random.default_rng(3)
    counts = rng.integers(0, 65, size=(24, 2)).astype(np.int32)
    counts[5, 1] = 0
    st = W.gen_stream(cfg, 24, counts=counts)
    if dyn:  # N3: hot set recomputed every 6 steps (each owner moves its own share)
        st = W.with_dynamic_hot(st, epoch=6)
    if layout:  # a random half of the rows first, in random order; the rest in id order
        order = np.random.default_rng(11).permutation(cfg.n_rows)[:cfg.n_rows // 2]
        st = W.dataclasses.replace(st, host_order=order.astype(np.int64))
    out = run_two_ranks(st, a2a=a2a, peer=peer)
    if peer:  # the variant actually served rows from the other rank's HBM
        assert out[0]["stats"]["gather_peer"] > 0 and out[1]["stats"]["gather_peer"] > 0
    o = Oracle(st)
    for s in range(st.steps):
        o.step()
        ref = o.schedule()
        urg = sorted(sum((out[r]["sched"][s]["urgent"].tolist() for r in range(2)), []))
        assert urg == ref["urgent"].tolist(), f"urgent differs at {s}"
        dfr = sorted(sum((list(zip(out[r]["sched"][s]["deferred"].tolist(),
                                   out[r]["sched"][s]["deferred_p"].tolist())) for r in range(2)), []))
        assert dfr == sorted(zip(ref["deferred"].tolist(), ref["deferred_p"].tolist())), f"deferred differs at {s}"
        age = sorted(sum((out[r]["sched"][s]["ageout"].tolist() for r in range(2)), []))
        assert age == ref["ageout"].tolist()
        xs = sorted(sum((out[r]["sched"][s]["transition"].tolist() for r in range(2)), []))
        assert xs == ref["transition"].tolist(), f"transition differs at {s}"
        for r in range(2):  # each rank only schedules rows it owns
            assert all(k % 2 == r for k in out[r]["sched"][s]["urgent"].tolist())
    ff = sorted(out[0]["ff"].tolist() + out[1]["ff"].tolist())
    assert ff == o.final_flush().tolist()
    lo = np.array([o.loss(s) for s in range(st.steps)])
    lg = out[0]["losses"] + out[1]["losses"]
    assert np.abs(lg - lo).max() <= 1e-5
    wo, Go = o.read_rows(np.arange(cfg.n_rows))
    assert np.abs(out[0]["w"] - wo).max() <= 1e-5
    assert np.abs(out[0]["G"] - Go).max() <= 1e-5
    assert o.violations == 0



@pytest.mark.parametrize("fused", [False, True])
def test_configs0_two_ranks_exact_shape(fused):
    """BASELINE.json configs[0] as stated: 1 table 10^4 x 16, batch 256, 20 steps, 2 GPUs
    (here: 2 rank processes sharing one B200), Zipf ids.  fused: the bench's default fused
    lookup (glue reads each rank's gathered distinct rows through its inverse index)."""
    from oracle.oracle import Oracle
    cfg = W.config("tiny")  # world 2, batch 256
    st = W.gen_stream(cfg, 20)
    out = run_two_ranks(st, fused=fused)
    o = Oracle(st)
    for s in range(st.steps):
        o.step()
        ref = o.schedule()
        urg = sorted(sum((out[r]["sched"][s]["urgent"].tolist() for r in range(2)), []))
        assert urg == ref["urgent"].tolist()
        dfr = sorted(sum((list(zip(out[r]["sched"][s]["deferred"].tolist(),
                                   out[r]["sched"][s]["deferred_p"].tolist())) for r in range(2)), []))
        assert dfr == sorted(zip(ref["deferred"].tolist(), ref["deferred_p"].tolist()))
    assert sorted(out[0]["ff"].tolist() + out[1]["ff"].tolist()) == o.final_flush().tolist()
    wo, Go = o.read_rows(np.arange(cfg.n_rows))
    assert np.array_equal(out[0]["w"], wo) and np.array_equal(out[0]["G"], Go)
    lo = np.array([o.loss(s) for s in range(st.steps)])
    assert np.abs(out[0]["losses"] + out[1]["losses"] - lo).max() <= 1e-5
