"""bench.py --gpus N (N > 1) under torchrun: one process per GPU, NCCL.

Weak scaling: in every step (= wave) each rank processes one GPU batch of
the cycled C2 stream; digests are routed to their owner GPU with NCCL
all-to-alls (rows A5-A8, see dist.py).  A dedup stream spans
ceil(batches / N) waves; tables are reset at every stream start.  The timed
region is bracketed by a barrier + device synchronisation and measured with
CUDA events; the maximum over ranks is reported.
"""
from __future__ import annotations

import json
import os

import numpy as np


def main(args, data, off):
    import torch
    import torch.distributed as dist

    import bench as B

    from . import dist as D

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist.init_process_group("nccl", device_id=dev)
    x = D.TorchDistExchange()
    plan = B.plan_batches(off)
    nb = len(plan)
    items_per_batch = max(j - k for k, j in plan)
    dd = D.DistDedup(x, local, B.BATCH_BYTES, B.BATCH_ITEMS + 1,
                     max(1 << 16, len(data) // 2048 // world))
    ddata = torch.from_numpy(data).to(dev)
    waves_per_stream = (nb + world - 1) // world

    def wave(w):
        if w % waves_per_stream == 0 and w > 0:
            dd.end_stream()
        b = ((w % waves_per_stream) * world + rank) % nb
        k, j = plan[b]
        seq = (w * world + rank) * items_per_batch
        out = dd.wave(ddata[int(off[k]):int(off[j])], off[k:j + 1] - off[k], seq)
        return int(off[j]) - int(off[k]), len(out.chunk_start)

    for w in range(args.warmup):
        wave(w)
    torch.cuda.synchronize()
    dist.barrier()
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    start.record()
    nbytes = nchunks = 0
    for w in range(args.warmup, args.warmup + args.steps):
        a, c = wave(w)
        nbytes += a
        nchunks += c
    end.record()
    torch.cuda.synchronize()
    dist.barrier()
    ms = torch.tensor([start.elapsed_time(end)], dtype=torch.float64, device=dev)
    tot = torch.tensor([nbytes, nchunks], dtype=torch.float64, device=dev)
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
                                   "1 MiB items, dup_frac 0.52, device-resident, one batch per "
                                   "GPU per step, digest all-to-all (NCCL) to owner GPUs",
                       "batch_bytes": B.BATCH_BYTES, "parallelism": f"{world} GPUs, "
                       "digest-prefix table sharding", "l2": "inputs larger than L2"},
            "gpu_launches": None,
        }
        print(json.dumps(line), flush=True)
    dd.close()
    dist.destroy_process_group()
