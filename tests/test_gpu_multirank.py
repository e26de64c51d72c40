"""world = 2: two rank processes and one POSIX-shm host table; mailboxes, flags and gates go
through host memory.  With >= 2 visible GPUs rank r runs on device r (the distinct-device
path: cross-GPU visibility of zero-copy host writes, NVLink peer loads, NCCL all-to-all);
the `same_device` variants put both ranks on device 0 (the only choice on a one-GPU box).
Compared against the oracle run with world 2: per-rank schedule sets (each rank owns
k mod 2 == rank), final flush, host table (w, G) and the global loss."""
import multiprocessing as mp
import os
import traceback

import numpy as np
import pytest

from paper_conf_asplos_xiezggl25_b200 import workload as W

pytestmark = pytest.mark.gpu


def n_gpus():
    import torch
    return torch.cuda.device_count()


def _rank_main(rank, st, shm, barrier, q, a2a=False, port=0, peer=False, fused=False, nonce=1, device=0,
               record=True, backend="gloo", gpu_drain=False, own_ids=False):
    try:
        import torch
        from paper_conf_asplos_xiezggl25_b200 import frugal as F
        from paper_conf_asplos_xiezggl25_b200.harness import A2ATrainer, Trainer, make_context
        torch.cuda.set_device(device)
        flags = (F.F_RECORD if record else F.F_TIMERS) | (F.F_A2A if a2a else 0) | (F.F_PEER if peer else 0) \
            | (F.F_GPU_DRAIN if gpu_drain else 0) | (F.F_OWN_IDS if own_ids else 0)
        fr = make_context(st, rank=rank, device=device, shm_name=shm, run_nonce=nonce, flags=flags)
        barrier.wait()
        if a2a:
            import torch.distributed as dist
            os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
            if backend == "nccl":
                dist.init_process_group("nccl", rank=rank, world_size=2, device_id=torch.device("cuda", device))
            else:
                dist.init_process_group("gloo", rank=rank, world_size=2)
            tr = A2ATrainer(fr, st, rank=rank, device=device, dist=dist, host_staging=backend == "gloo")
        else:
            # record=False: the bench's configuration -- no per-step synchronisation, inputs in HBM
            tr = Trainer(fr, st, rank=rank, device=device, fused_lookup=fused, device_inputs=not record)
        sched = []
        for s in range(st.steps):
            got = {}

            def cb(s_):
                got.update(fr.get_schedule())
                got["transition"] = fr.get_transition()
            tr.step(on_schedule=cb if record else None)
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


def run_two_ranks(st, timeout=600, a2a=False, peer=False, fused=False, same_device=True, record=True,
                  backend="gloo", gpu_drain=False, own_ids=False):
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
    if not same_device and n_gpus() < 2:
        pytest.skip("needs 2 GPUs (rank r on device r)")
    ps = [ctx.Process(target=_rank_main, args=(r, st, shm, barrier, q, a2a, port, peer, fused, nonce,
                                               0 if same_device else r, record, backend, gpu_drain, own_ids))
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


@pytest.mark.parametrize("same_device", [True, False])
@pytest.mark.parametrize("opt,a2a,peer,dyn,layout", [("adagrad", False, False, False, False),
                                                     ("sgd", False, False, False, False),
                                                     ("adagrad", True, False, False, False),
                                                     ("adagrad", False, True, False, False),
                                                     ("adagrad", False, False, True, False),
                                                     ("adagrad", False, False, False, True)])
def test_two_ranks_parity(opt, a2a, peer, dyn, layout, same_device):
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
    out = run_two_ranks(st, a2a=a2a, peer=peer, same_device=same_device)
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



@pytest.mark.parametrize("same_device", [True, False])
@pytest.mark.parametrize("fused", [False, True])
def test_configs0_two_ranks_exact_shape(fused, same_device):
    """BASELINE.json configs[0] as stated: 1 table 10^4 x 16, batch 256, 20 steps, 2 GPUs
    (here: 2 rank processes sharing one B200), Zipf ids.  fused: the bench's default fused
    lookup (glue reads each rank's gathered distinct rows through its inverse index)."""
    from oracle.oracle import Oracle
    cfg = W.config("tiny")  # world 2, batch 256
    st = W.gen_stream(cfg, 20)
    out = run_two_ranks(st, fused=fused, same_device=same_device)
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


def _compare_whole_run(st, out, exact=True):
    """Values-only comparison (no per-step sets): losses, final flush, host table."""
    from oracle.oracle import Oracle
    o = Oracle(st)
    o.run()
    assert o.violations == 0
    lo = np.array([o.loss(s) for s in range(st.steps)])
    assert np.abs(out[0]["losses"] + out[1]["losses"] - lo).max() <= 1e-5
    assert sorted(out[0]["ff"].tolist() + out[1]["ff"].tolist()) == o.final_flush().tolist()
    wo, Go = o.read_rows(np.arange(st.cfg.n_rows))
    if exact:
        assert np.array_equal(out[0]["w"], wo) and np.array_equal(out[0]["G"], Go)
    assert np.abs(out[0]["w"] - wo).max() <= 1e-5 and np.abs(out[0]["G"] - Go).max() <= 1e-5


@pytest.mark.parametrize("same_device", [True, False])
@pytest.mark.parametrize("fused", [False, True])
def test_two_ranks_overlapped_pipeline(fused, same_device):
    """world 2 in the bench's configuration (F_TIMERS only, device-resident inputs,
    no per-step callbacks, so ingest, drain, mailbox exchange and gates overlap freely);
    losses, final-flush set and the whole host table against the oracle."""
    cfg = W.config("tiny", world=2, batch=128, lookahead=4, age_out=3)
    st = W.gen_stream(cfg, 60)
    out = run_two_ranks(st, fused=fused, same_device=same_device, record=False)
    _compare_whole_run(st, out)


@pytest.mark.parametrize("variant", ["p2f", "peer", "a2a_gloo", "a2a_nccl"])
@pytest.mark.parametrize("same_device", [True, False])
def test_two_ranks_100_step_stress(variant, same_device):
    """100 steps of configs[0] (world 2, batch 256, L 10, D 10) for the host-bounced P2F path,
    the N4 peer variant and the a2a comparison path (gloo with host staging, or NCCL -- over
    NVLink when the ranks sit on distinct GPUs; NCCL needs distinct devices).  Every schedule
    set per step, the oracle's invariant (2), losses, final flush and the whole table."""
    if variant == "a2a_nccl" and same_device:
        pytest.skip("NCCL needs one device per rank")
    from oracle.oracle import Oracle
    cfg = W.config("tiny")
    st = W.gen_stream(cfg, 100)
    out = run_two_ranks(st, a2a=variant.startswith("a2a"), peer=variant == "peer", same_device=same_device,
                        backend="nccl" if variant == "a2a_nccl" else "gloo", timeout=1200)
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
        assert age == ref["ageout"].tolist(), f"age-out differs at {s}"
        assert any(out[r]["sched"][s]["gate_wait"] for r in range(2)) == ref["gate_wait"]
    assert o.violations == 0
    assert sorted(out[0]["ff"].tolist() + out[1]["ff"].tolist()) == o.final_flush().tolist()
    lo = np.array([o.loss(s) for s in range(st.steps)])
    assert np.abs(out[0]["losses"] + out[1]["losses"] - lo).max() <= 1e-5
    wo, Go = o.read_rows(np.arange(cfg.n_rows))
    assert np.array_equal(out[0]["w"], wo) and np.array_equal(out[0]["G"], Go)
    if variant == "peer":
        assert out[0]["stats"]["gather_peer"] > 0 and out[1]["stats"]["gather_peer"] > 0


@pytest.mark.parametrize("record", [True, False])
@pytest.mark.parametrize("same_device", [True, False])
def test_two_ranks_gpu_drain(record, same_device):
    """FRUGAL_F_GPU_DRAIN at world 2 (the default drain's flushing threads publish each owner's
    FLAG_SIDE_FIRST from the host; here the drain kernel does, after its zero-copy scatter)."""
    from oracle.oracle import Oracle
    cfg = W.config("tiny", world=2, batch=128, lookahead=4, age_out=3)
    st = W.gen_stream(cfg, 50)
    out = run_two_ranks(st, same_device=same_device, record=record, gpu_drain=True, fused=True)
    if record:
        o = Oracle(st)
        for s in range(st.steps):
            o.step()
            ref = o.schedule()
            dfr = sorted(sum((list(zip(out[r]["sched"][s]["deferred"].tolist(),
                                       out[r]["sched"][s]["deferred_p"].tolist())) for r in range(2)), []))
            assert dfr == sorted(zip(ref["deferred"].tolist(), ref["deferred_p"].tolist())), f"deferred differs at {s}"
    _compare_whole_run(st, out)


@pytest.mark.parametrize("variant", ["p2f", "peer", "a2a", "overlapped", "dyn"])
def test_two_ranks_own_ids(variant):
    """Ingest v2 (FRUGAL_F_OWN_IDS): every rank gets only its own ids; the ranks exchange their
    distinct ids, grouped by owner, through the host id mailbox, and each owner merges the ids
    it owns into its read sets -- every set per step, losses and the whole table as the oracle."""
    from oracle.oracle import Oracle
    cfg = W.config("tiny", world=2, batch=96, lookahead=4, age_out=3)
    rng = np.random.default_rng(21)
    counts = rng.integers(0, 97, size=(40, 2)).astype(np.int32)
    counts[7, 0] = 0
    counts[9] = 0
    st = W.gen_stream(cfg, 40, counts=counts)
    if variant == "dyn":
        st = W.with_dynamic_hot(st, epoch=6)
    record = variant != "overlapped"
    out = run_two_ranks(st, a2a=variant == "a2a", peer=variant == "peer", record=record, own_ids=True,
                        fused=variant == "overlapped")
    if record:
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
    _compare_whole_run(st, out)
