"""world_size-2 gloo tests on CPU of the multi-rank host logic: the bench's max-over-ranks
timing, the per-rank input slicing, and that every rank generates the same seeded stream
(each rank enqueues the ids of ALL ranks, so they must agree bit for bit)."""
import os
import socket

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import bench
    from paper_conf_asplos_xiezggl25_b200 import workload as W
    mx = bench.dist_max(float(10 + rank), world, dist)
    cfg = W.config("tiny", world=world, batch=64)
    st = W.gen_stream(cfg, 6)
    h = torch.tensor([int(np.bitwise_xor.reduce(st.ids.ravel().astype(np.int64)))], dtype=torch.int64)
    hs = [torch.zeros_like(h) for _ in range(world)]
    dist.all_gather(hs, h)
    mine = np.ascontiguousarray(st.x[:, rank])
    assert mine.shape == (6, 64, 16)
    q.put((rank, mx, [int(x) for x in hs], float(np.abs(mine).sum())))
    dist.destroy_process_group()


def test_gloo_world2_bench_helpers():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = [q.get(timeout=120) for _ in range(world)]
    for p in ps:
        p.join(timeout=30)
    out.sort()
    assert all(o[1] == 11.0 for o in out)             # max over ranks
    assert out[0][2] == out[1][2] and out[0][2][0] == out[0][2][1]  # same stream on every rank
    assert out[0][3] != out[1][3]                     # each rank takes its own dense inputs
