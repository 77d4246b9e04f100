"""bench.py --gpus N (N > 1) under torchrun: one process per GPU, NCCL.

Weak scaling: in every step (= wave) each rank processes one 64 MiB GPU
batch of the cycled C2 stream (the single-GPU step); digests are routed to
their owner GPU over NCCL (rows A5-A8) by the C++ wave pipeline
(csrc/dist.cpp, dist.NativeWavePipeline): `DEPTH` waves are in flight per
rank, so a rank's GPU keeps chunking and hashing later waves while the
exchange of the oldest one runs.  A dedup stream spans max(batches / N,
4 * DEPTH) waves; the table shards are reset at every stream start (later
passes over the cycled stream inside one stream are duplicates).  The timed region is bracketed by a
barrier + device synchronisation and measured with CUDA events; the maximum
over ranks is reported.
"""
from __future__ import annotations

import json
import os


# waves in flight per rank and SHA-1 bytes per lane of a wave.  Measured
# (world 1, 64 MiB waves, early counts, graphs primed;
# profiles/r01_dist_depth_lane_sweep.txt): depth 24 / 16 KiB 632-643 GB/s;
# 24 / 32 KiB 606-632; 32 / 8 KiB 578; 24 / 8 KiB 578; 16 / 16 KiB 593-595;
# 16 / 8 KiB 570; 16 / 32 KiB 501-503; 12 / 8 KiB 524; 8 / 8 KiB 400
DEPTH = int(os.environ.get("DEDUP_DIST_DEPTH", "24"))
SHA_LANE_BYTES = int(os.environ.get("DEDUP_DIST_SHA_LANE", "16384"))
# end_stream without draining the waves in flight (the table reset goes in
# before the next stream's first wave on the owner stream)
DRAIN = os.environ.get("DEDUP_DIST_DRAIN", "0") != "0"


def main(args, data, off, B):
    """B: the running bench module (batch settings, plan_batches, metric)."""
    import torch
    import torch.distributed as dist

    from . import dist as D

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist.init_process_group("nccl", device_id=dev)
    plan = B.plan_batches(off)
    nb = len(plan)
    items_per_batch = max(j - k for k, j in plan)
    wave_bytes = B.BATCH_BYTES
    idt = torch.zeros(128, dtype=torch.uint8, device=dev)
    if rank == 0:
        idt.copy_(torch.frombuffer(bytearray(D.nccl_unique_id()), dtype=torch.uint8))
    dist.broadcast(idt, 0)
    pipe = D.NativeWavePipeline(bytes(idt.cpu().numpy()), world, rank, local, wave_bytes,
                                items_per_batch + 1,
                                max(1 << 16, len(data) // 2048 // world), depth=DEPTH,
                                sha_lane_bytes=SHA_LANE_BYTES)
    ddata = torch.from_numpy(data).to(dev)
    # A table reset completes every wave in flight first (end_stream), so a
    # dedup stream spans at least 4 pipeline depths of waves (the C2 batches
    # cycled; later passes over the data inside one stream are duplicates).
    waves_per_stream = max((nb + world - 1) // world, 4 * DEPTH)
    counted = {"bytes": 0, "chunks": 0}

    def take(outs, timed):
        for nbytes, nchunks in outs:   # results stay in pinned host memory
            if timed:
                counted["bytes"] += int(nbytes)
                counted["chunks"] += int(nchunks)

    def wave(w, timed):
        if w % waves_per_stream == 0 and w > 0:
            take(pipe.end_stream(collect=False, drain=DRAIN), timed)
        b = ((w % waves_per_stream) * world + rank) % nb
        k, j = plan[b]
        seq = (w * world + rank) * items_per_batch
        take(pipe.submit([(ddata[int(off[k]):int(off[j])], off[k:j + 1] - off[k], seq)],
                         collect=False), timed)

    # Setup (untimed, before the W warm-up steps): one dedup stream of
    # waves_per_stream waves visits every (slot, batch geometry) pair the
    # timed waves use (slot = w % DEPTH, batch = (w * N + rank) % nb; all of
    # them whenever lcm(DEPTH, nb) <= waves_per_stream, e.g. C2's 3 batches
    # at depth 24: 24 <= 96), so each slot's
    # local-row CUDA graphs are captured here, not inside the timed region;
    # then a fresh table.
    for w in range(waves_per_stream):
        wave(w, False)
    take(pipe.end_stream(collect=False), False)
    for w in range(args.warmup):
        wave(w, False)
    take(pipe.flush(collect=False), False)
    torch.cuda.synchronize()
    dist.barrier()
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    start.record()
    for w in range(args.warmup, args.warmup + args.steps):
        wave(w, True)
    take(pipe.flush(collect=False), True)
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
                                   "1 MiB items, dup_frac 0.52, device-resident, one 64 MiB "
                                   "batch per GPU per step, digest exchange (NCCL send/recv, "
                                   "C++ wave pipeline) to owner GPUs",
                       "batch_bytes": wave_bytes, "waves_in_flight": DEPTH,
                       "parallelism": f"{world} GPUs, digest-prefix table sharding",
                       "l2": "inputs larger than L2"},
            "gpu_launches": None,
        }
        print(json.dumps(line), flush=True)
    pipe.close()
    dist.destroy_process_group()
