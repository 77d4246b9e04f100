"""Multi-rank (world_size 2) CPU tests of the host side of bench.py --gpus N
(paper_conf_ipps_rockenbachsgmtd19_b200/dist_bench.py) over torch.distributed
with the gloo backend: the pass plan, every rank's wave schedule and sequence
numbers, the NCCL-id broadcast and the cross-rank reduction of the timed
region.  The device pipeline itself (csrc/mg.cpp) is tested on the GPU at
G = 1..8 logical ranks (tests/test_gpu_mg.py) and through NCCL at world 1
(tests/test_gpu_dist_loopback.py)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synthgen
from paper_conf_ipps_rockenbachsgmtd19_b200 import dist_bench as DB

MiB = 1 << 20


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, fn_name, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        q.put((rank, globals()[fn_name](rank, world)))
    except Exception as e:  # surface the failure to the parent
        q.put((rank, e))
    finally:
        dist.destroy_process_group()


def _run(fn_name, world=2):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, fn_name, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = dict(q.get(timeout=300) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    for r, v in out.items():
        if isinstance(v, Exception):
            raise v
    return out


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("n_items,item", [(672, MiB), (10, MiB), (5, MiB), (1, 1000)])
def test_pass_plan(world, n_items, item):
    """A multiple of world batches of consecutive whole items covering the
    stream once, each within the byte / item bounds, balanced."""
    off = np.minimum(np.arange(n_items + 1, dtype=np.uint64) * item, n_items * item)
    plan = DB.pass_plan(off, world, 64 * MiB, 64)
    assert len(plan) % world == 0
    assert plan[0][0] == 0 and plan[-1][1] == n_items
    assert all(a[1] == b[0] for a, b in zip(plan, plan[1:]))
    sizes = [j - k for k, j in plan]
    assert max(sizes) - min(sizes) <= 1
    assert all(int(off[j]) - int(off[k]) <= 64 * MiB and j - k <= 64 for k, j in plan)
    if n_items == 672:
        assert len(plan) == {1: 11, 2: 12, 3: 12, 4: 12, 8: 16}[world]


def _schedule_case(rank, world):
    """Every rank derives its schedule alone; gathered, the schedules give
    every item of every pass exactly once, in seq order by (wave, rank), and
    every rank has the same number of waves (NCCL matches calls in order)."""
    off = synthgen.split_items(np.zeros(37 * MiB + 5, np.uint8), MiB)
    n_items = len(off) - 1
    plan = DB.pass_plan(off, world, 8 * MiB, 8)
    mine = [DB.rank_schedule(plan, world, rank, p, n_items) for p in range(3)]
    got = [None] * world
    dist.all_gather_object(got, mine)
    out = []
    for p in range(3):
        assert len({len(g[p]) for g in got}) == 1
        waves = len(got[0][p])
        for v in range(waves):
            for r in range(world):
                wv, k, j, seq = got[r][p][v]
                assert wv == v and seq == p * n_items + k
                out.extend(range(seq, seq + (j - k)))
    assert out == list(range(3 * n_items))
    return len(plan)


def test_rank_schedule_gloo():
    out = _run("_schedule_case")
    assert out[0] == out[1]


def _id_and_reduce_case(rank, world):
    payload = bytes(range(128)) if rank == 0 else None
    got = DB.broadcast_bytes(payload, torch.device("cpu"))
    assert got == bytes(range(128))
    ms, counts = DB.reduce_timed(10.0 + rank, [100 * (rank + 1), 7], torch.device("cpu"))
    return ms, counts


def test_nccl_id_broadcast_and_reduction_gloo():
    out = _run("_id_and_reduce_case")
    for r in range(2):
        ms, counts = out[r]
        assert ms == 11.0                   # max over ranks
        assert counts == [300.0, 14.0]      # sums over ranks
