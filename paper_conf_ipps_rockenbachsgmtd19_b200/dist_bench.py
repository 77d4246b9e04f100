"""bench.py --gpus N (N > 1) under torchrun: one process per GPU, NCCL.

Weak scaling on the headline workload (BASELINE.json configs[2]: the
672 MiB native-sized stream C3 "at 1/2/4/8 GPUs with all-to-all digest
routing"): a pass is one pass over the whole C3 stream as a new dedup
stream, its items cut into a multiple of N GPU batches (<= 64 MiB, whole
items, balanced) that go to the ranks round-robin -- wave v of a pass holds
batches vN .. vN + N - 1, one per rank; a step is N passes, so every GPU
processes one stream's worth (672 MiB) per step at any N, as the single-GPU
step does.  Every rank runs the C++ wave
pipeline of the multi-GPU engine (csrc/mg.cpp through dedup_dist_*,
dist.NativeWavePipeline): local rows of up to DEPTH waves in flight, digests
routed to their owner rank over NCCL (rows A5-A8).  Consecutive passes run
back to back (the table reset of a new stream is deferred to its first
wave, no drain).  The timed region is bracketed by a barrier + device
synchronisation, measured with CUDA events after dedup_dist_join (every
completed wave's results), and the maximum over ranks is reported; `value`
= the stream bytes of all K passes / that time.

The host-side pieces (pass plan, per-rank schedule, sequence numbers, the
NCCL id broadcast and the cross-rank reduction) are plain functions, tested
with the gloo backend at world size 2 (tests/test_dist_gloo.py).
"""
from __future__ import annotations

import json
import os
import time

import numpy as np

# waves in flight per rank and SHA-1 bytes per lane of a wave (measured at
# world size 1, profiles/r01_dist_depth_lane_sweep.txt: depth 24 / 16 KiB)
DEPTH = int(os.environ.get("DEDUP_DIST_DEPTH", "24"))
SHA_LANE_BYTES = int(os.environ.get("DEDUP_DIST_SHA_LANE", "16384"))


def pass_plan(off, world: int, batch_bytes: int, batch_items: int):
    """Batches (item ranges [k, j)) of one pass over the stream: the fewest
    multiple of `world` batches of consecutive whole items, balanced by item
    count, each within batch_bytes / batch_items."""
    n_items = len(off) - 1
    nb = world * max(1, -(-max(1, n_items) // (world * batch_items)))
    while True:
        b = [(n_items * i) // nb for i in range(nb + 1)]
        plan = [(b[i], b[i + 1]) for i in range(nb)]
        if all(int(off[j]) - int(off[k]) <= batch_bytes and j - k <= batch_items
               for k, j in plan):
            return plan
        nb += world


def rank_schedule(plan, world: int, rank: int, pass_index: int, n_items: int):
    """(wave, k, j, first_seq) of this rank's batches in one pass: wave v
    takes batch v * world + rank; items are numbered across passes, so pass
    p's item k has seq p * n_items + k."""
    out = []
    for v in range(len(plan) // world):
        k, j = plan[v * world + rank]
        out.append((v, k, j, pass_index * n_items + k))
    return out


def broadcast_bytes(payload: bytes | None, device, src: int = 0) -> bytes:
    """rank `src`'s payload (e.g. the 128-byte NCCL id) on every rank."""
    import torch
    import torch.distributed as dist
    n = torch.zeros(1, dtype=torch.int64, device=device)
    if dist.get_rank() == src:
        n[0] = len(payload)
    dist.broadcast(n, src)
    t = torch.zeros(int(n.item()), dtype=torch.uint8, device=device)
    if dist.get_rank() == src:
        t.copy_(torch.frombuffer(bytearray(payload), dtype=torch.uint8))
    dist.broadcast(t, src)
    return bytes(t.cpu().numpy())


def reduce_timed(ms: float, counts, device):
    """(max over ranks of ms, sum over ranks of each count)."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([ms], dtype=torch.float64, device=device)
    c = torch.tensor([float(x) for x in counts], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    dist.all_reduce(c, op=dist.ReduceOp.SUM)
    return float(t.item()), [float(x) for x in c.tolist()]


def main(args, data, off, B):
    """B: the running bench module (workload settings, metric, helpers)."""
    import torch
    import torch.distributed as dist

    from . import dist as D

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist.init_process_group("nccl", device_id=dev)
    n_items = len(off) - 1
    plan = pass_plan(off, world, B.BATCH_BYTES, B.BATCH_ITEMS)
    items_per_batch = max(j - k for k, j in plan)
    wave_bytes = max(int(off[j]) - int(off[k]) for k, j in plan)
    nccl_id = broadcast_bytes(D.nccl_unique_id() if rank == 0 else None, dev)
    pipe = D.NativeWavePipeline(nccl_id, world, rank, local, wave_bytes, items_per_batch + 1,
                                max(1 << 16, len(data) // 2048 // world), depth=DEPTH,
                                sha_lane_bytes=SHA_LANE_BYTES)
    ddata = torch.from_numpy(data).to(dev)
    views = {(k, j): ddata[int(off[k]):int(off[j])] for k, j in plan}
    counted = {"bytes": 0, "chunks": 0}

    def take(outs, timed):
        for nbytes, nchunks in outs:   # results stay in pinned host memory
            if timed:
                counted["bytes"] += int(nbytes)
                counted["chunks"] += int(nchunks)

    def run_step(st, timed, submit_one):  # N passes: one stream's worth per GPU
        for p in range(st * world, (st + 1) * world):
            run_pass(p, timed, submit_one)

    def run_pass(p, timed, submit_one):
        take(pipe.end_stream(collect=False, drain=False), timed)   # new dedup stream
        for _, k, j, seq in rank_schedule(plan, world, rank, p, n_items):
            take(submit_one(k, j, seq), timed)

    def sub_device(k, j, seq):
        return pipe.submit([(views[(k, j)], off[k:j + 1] - off[k], seq)], collect=False)

    def timed_run(submit_one, steps):
        for st in range(args.warmup):
            run_step(st, False, submit_one)
        take(pipe.flush(collect=False), False)
        torch.cuda.synchronize()
        dist.barrier()
        counted["bytes"] = counted["chunks"] = 0
        l0, a0 = pipe.kernel_launches(), pipe.a2a_bytes()
        start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        start.record()
        for st in range(args.warmup, args.warmup + steps):
            run_step(st, True, submit_one)
        take(pipe.flush(collect=False), True)
        pipe.join()
        end.record()
        torch.cuda.synchronize()
        dist.barrier()
        return reduce_timed(start.elapsed_time(end),
                            [counted["bytes"], counted["chunks"], pipe.kernel_launches() - l0,
                             pipe.a2a_bytes() - a0], dev)

    # untimed priming pass: every slot's graph and the NCCL channels set up
    run_pass(0, False, sub_device)
    take(pipe.flush(collect=False), False)
    clk = B.ClockSampler(local)
    with clk:
        t, (tot_bytes, tot_chunks, launches, a2a) = timed_run(sub_device, args.steps)
    # ---- e2e: the same passes with every batch copied H2D from pinned host
    # memory on the producer stream inside the timed region ----
    mine = [(k, j) for v, k, j, _ in rank_schedule(plan, world, rank, 0, n_items)]
    pin = {kj: torch.from_numpy(data[int(off[kj[0]]):int(off[kj[1]])]).pin_memory()
           for kj in mine}
    ring = [torch.empty(wave_bytes + 256, dtype=torch.uint8, device=dev)
            for _ in range(DEPTH + 2)]
    cur = {"i": 0}

    def sub_host(k, j, seq):
        buf = ring[cur["i"] % len(ring)]
        cur["i"] += 1
        n = int(off[j]) - int(off[k])
        buf[:n].copy_(pin[(k, j)], non_blocking=True)
        return pipe.submit([(buf[:n], off[k:j + 1] - off[k], seq)], collect=False)

    e2e_steps = max(3, min(args.steps, 10))
    te, (e_bytes, e_chunks, _, _) = timed_run(sub_host, e2e_steps)
    pipe.close()
    line = None
    if rank == 0:
        value = tot_bytes / (t / 1e3) / 1e9
        line = {
            "metric": B.METRIC, "value": value, "unit": "GB/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": t / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "chunks_per_s": tot_chunks / (t / 1e3),
            "config": {"workload": B.WORKLOAD_DESC + f"; at N GPUs a step is N such passes "
                                                     f"(each a new dedup stream), a pass split "
                                                     f"into {len(plan)} batches, "
                                                     f"{len(plan) // world} waves of one batch "
                                                     "per GPU",
                       "batch_bytes": wave_bytes, "waves_in_flight": DEPTH,
                       "parallelism": f"{world} GPUs (one process each), digest-prefix table "
                                      "sharding, NCCL grouped send/recv (C++ engine)",
                       "l2": "inputs larger than L2 (672 MiB stream)"},
            "clocks": clk.summary(), "gpu_launches": int(launches),
            # rows A6 + A8 over NVLink: bytes that left each GPU per second,
            # against NVLink5's 900 GB/s per direction per GPU (nominal)
            "a2a": {"bytes_per_step": a2a / args.steps,
                    "gbs_per_gpu": a2a / world / (t / 1e3) / 1e9,
                    "nvlink_frac": a2a / world / (t / 1e3) / 1e9 / 900.0,
                    "peak_source": "nominal NVLink5 900 GB/s per direction per GPU"},
            "e2e": {"value": e_bytes / (te / 1e3) / 1e9, "unit": "GB/s",
                    "h2d_bytes_per_step": e_bytes / e2e_steps,
                    "d2h_bytes_per_step": 33 * e_chunks / e2e_steps, "steps": e2e_steps,
                    "api": "dedup_dist_submit after a pinned H2D copy of each batch on the "
                           "producer stream; results in mapped pinned memory"},
        }
    # ---- per-kernel roofline (rank 0, the GPU otherwise idle) + CPU baseline ----
    dist.barrier()
    if rank == 0:
        rates = B.int_rates()
        int_peak = B.sha1_peak(rates)
        iso = B.isolated_kernels(ddata, off, int_peak, rates["lop3"])
        kd = iso["sha1"]
        line["roofline"] = {"kernel": "sha1_kernel", "bound": "alu", "achieved": kd["achieved"],
                            "peak": int_peak, "unit": "Tops/s", "frac": kd["achieved"] / int_peak,
                            "traffic": None, "peak_source": "measured (dedup_probe_int_rates)",
                            "note": "isolated full-GPU SHA-1 launches on rank 0's GPU"}
        line["kernels"] = {"sha1": kd, "chunk_stage": iso["chunk_stage"],
                           "int_rates_tops": rates}
        if not args.no_cpu_baseline:
            line["cpu_baseline"] = B.cpu_baseline(data, off)
        print(json.dumps(line), flush=True)
    dist.barrier()
    dist.destroy_process_group()
    time.sleep(0.1)
