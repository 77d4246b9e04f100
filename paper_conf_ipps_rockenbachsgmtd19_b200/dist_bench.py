"""bench.py --gpus N (N > 1) under torchrun: one process per GPU, NCCL.

Weak scaling: in every step (= wave) each rank processes one pass over the
whole C2 stream (184 MiB, 184 items of 1 MiB) as one GPU batch; digests are
routed to their owner GPU with NCCL all-to-alls (rows A5-A8, see dist.py).
Waves are pipelined (dist.WavePipeline): `DEPTH` waves are in flight per
rank, so a rank's GPU keeps chunking and hashing later waves while the
exchange of the oldest one runs.  The wave is the whole stream because the
pipeline's host orchestration costs ~1 ms per wave.
A dedup stream spans 4 * DEPTH waves; the table shards are reset at every
stream start (every rank passes over the same bytes, so within a stream
the other ranks' and later passes' chunks are duplicates).  The timed region is bracketed by a
barrier + device synchronisation and measured with CUDA events; the maximum
over ranks is reported.
"""
from __future__ import annotations

import json
import os

import numpy as np

DEPTH = 4  # waves in flight per rank


def main(args, data, off, B):
    """B: the running bench module (batch settings, plan_batches, metric)."""
    import torch
    import torch.distributed as dist

    from . import dist as D
    from .api import Dedup

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist.init_process_group("nccl", device_id=dev)
    x = D.TorchDistExchange()
    n_items = len(off) - 1
    plan = [(0, n_items)]                # one wave batch = the whole stream
    nb = 1
    items_per_batch = n_items
    wave_bytes = int(off[-1])
    # the owner receives up to `world` batches' records per wave
    owner = Dedup(local, batch_bytes=min(1 << 30, world * wave_bytes), batch_items=1, slots=1,
                  table_capacity=max(1 << 16, len(data) // 2048 // world), host_fed=False,
                  owner_rank=rank, num_owners=world)
    pipe = D.WavePipeline(x, [owner], local, wave_bytes, n_items + 1, depth=DEPTH)
    ddata = torch.from_numpy(data).to(dev)
    # A table reset completes every wave in flight first (end_stream), so a
    # dedup stream spans at least 4 pipeline depths of waves (the C2 batches
    # cycled; later passes over the data inside one stream are duplicates).
    waves_per_stream = 4 * DEPTH
    counted = {"bytes": 0, "chunks": 0}

    def take(outs, timed):
        for wave in outs:
            o = wave[0]
            if timed:
                counted["bytes"] += int(np.sum(o.item_len))
                counted["chunks"] += len(o.chunk_start)

    def wave(w, timed):
        if w % waves_per_stream == 0 and w > 0:
            take(pipe.end_stream(), timed)
        b = ((w % waves_per_stream) * world + rank) % nb
        k, j = plan[b]
        seq = (w * world + rank) * items_per_batch
        take(pipe.submit([(ddata[int(off[k]):int(off[j])], off[k:j + 1] - off[k], seq)]),
             timed)

    for w in range(args.warmup):
        wave(w, False)
    take(pipe.flush(), False)
    torch.cuda.synchronize()
    dist.barrier()
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    start.record()
    for w in range(args.warmup, args.warmup + args.steps):
        wave(w, True)
    take(pipe.flush(), True)
    end.record()
    torch.cuda.synchronize()
    dist.barrier()
    ms = torch.tensor([start.elapsed_time(end)], dtype=torch.float64, device=dev)
    tot = torch.tensor([counted["bytes"], counted["chunks"]], dtype=torch.float64, device=dev)
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    dist.all_reduce(tot, op=dist.ReduceOp.SUM)
    t = float(ms.item())
    if rank == 0:
        line = {
            "metric": B.METRIC, "value": float(tot[0]) / (t / 1e3) / 1e9, "unit": "GB/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": t / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "chunks_per_s": float(tot[1]) / (t / 1e3),
            "config": {"workload": f"{B.WORKLOAD}: 184 MiB simlarge-sized synthetic stream, "
                                   "1 MiB items, dup_frac 0.52, device-resident, one pass over "
                                   "the stream per GPU per step, digest all-to-all (NCCL) to "
                                   "owner GPUs",
                       "batch_bytes": wave_bytes, "waves_in_flight": DEPTH,
                       "parallelism": f"{world} GPUs, digest-prefix table sharding",
                       "l2": "inputs larger than L2"},
            "gpu_launches": None,
        }
        print(json.dumps(line), flush=True)
    pipe.close()
    owner.close()
    dist.destroy_process_group()
