#!/usr/bin/env python
"""Benchmark of the GPU Dedup hot path (Rabin CDC -> SHA-1 -> global dedup).

Contract (README / DESIGN.md "Measurement"):
  python bench.py --gpus N --steps K --warmup W [--impl b200|reference]
prints ONE JSON line on rank 0.

A step is one pass of the whole hot path (rows A1-A9 of SURVEY 8(a)) over
one GPU batch of the BASELINE.json configs[1] workload: the 184 MiB
simlarge-sized synthetic stream (1 MiB items, ~50 % duplicate chunks),
cycled; at every wrap of the stream a new dedup stream (fresh digest table)
starts.  `value` is input GB/s (1e9 B/s) with the stream resident in HBM
(device-timed with CUDA events around submit..drain); `e2e` is the same
metric through dedup_submit_batch with pinned HOST buffers (H2D and the
result read-back inside the timed region).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

# Up to 32 hardware work queues, so that the engine's per-slot streams run
# concurrently (must be set before CUDA is initialised).
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
# per-stage CUDA-event times are read for every 8th batch (event queries cost
# host time); the roofline uses those samples
os.environ.setdefault("DEDUP_TIME_EVERY", "8")

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import synthgen  # noqa: E402

MiB = 1 << 20
ITEM_BYTES = MiB                 # the paper's fixed 1 MB batches
BATCH_BYTES = 64 * MiB           # GPU batch (step); C2 batch sweep 1-64 MiB
BATCH_ITEMS = 64
SLOTS = 40                       # batches in flight ("memory spaces")
WORKLOAD = "C2"
METRIC = "input GB/s & chunks/s (dedup hot path) at 1/2/4/8 B200; % of HBM/INT roofline"

# SHA-1 algorithmic 32-bit integer ops per 64-byte block (FIPS 180-4 6.1.2,
# counting a 3-input logic/add as one op and a rotate as one op):
#   80 rounds x (f 1 + rotl5 1 + adds 2 + rotl30 1) + 64 x schedule 3 + 5.
SHA1_OPS_PER_BLOCK = 80 * 5 + 64 * 3 + 5
SHA1_ALU_OPS_PER_BLOCK = 80 * 3 + 64 * 3       # of which on the ALU pipe
# Rabin rolling step per input byte: 2 table lookups, shift-in,
# 2 address formations, 1 3-way XOR, test + bit = 8 ops.
SCAN_OPS_PER_BYTE = 8
# Integer-op peak = instruction issue: 148 SM x 4 SMSP x 1 warp-instr/clk x 32
# lanes (B300_MICROARCH.md: 4 SMSPs, ALU and FMA pipes 16 lanes/clk each per
# SMSP, so a mix of ALU-pipe and IMAD ops can fill every issue slot).
INT_LANES_PER_SM_CLK = 128


def h2d_bandwidth(pin, dev, nbytes=64 * MiB, reps=10):
    """Plain pinned host -> device copy bandwidth (the e2e roofline, PCIe)."""
    import torch
    src = torch.from_numpy(pin[:nbytes])
    dst = dev[:nbytes]
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    dst.copy_(src, non_blocking=True)
    torch.cuda.synchronize()
    ev[0].record()
    for _ in range(reps):
        dst.copy_(src, non_blocking=True)
    ev[1].record()
    ev[1].synchronize()
    return nbytes * reps / (ev[0].elapsed_time(ev[1]) * 1e-3) / 1e9


def engine_kwargs(stream_bytes: int) -> dict:
    return dict(batch_bytes=BATCH_BYTES, batch_items=BATCH_ITEMS, slots=SLOTS,
                table_capacity=max(1 << 16, stream_bytes // 2048), host_fed=True)


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured"
    return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback"


class ClockSampler:
    """NVML sampling of SM clock + throttle reasons during the timed region."""

    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
        0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
        0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
        0x100: "display_clock_setting"}

    def __init__(self, device: int):
        self.samples, self.reasons, self._stop = [], set(), threading.Event()
        self.max_mhz = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and bit != 0x1:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.005)

    def __enter__(self):
        if self.nv is not None:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv is not None:
            self._t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                    "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def plan_batches(off):
    out, k, n = [], 0, len(off) - 1
    while k < n:
        j = k + 1
        while j < n and j - k < BATCH_ITEMS and int(off[j + 1]) - int(off[k]) <= BATCH_BYTES:
            j += 1
        out.append((k, j))
        k = j
    return out


def run_steps(d, submit, n_batches, steps, first_step):
    """Submit `steps` consecutive steps (batches, cycling the stream)."""
    for s in range(first_step, first_step + steps):
        b = s % n_batches
        if b == 0 and s > 0:
            d.end_stream()
        while True:
            try:
                submit(b)
                break
            except Exception as e:
                if "EAGAIN" not in str(e):
                    raise
                # a non-blocking drain first releases the slots handed out by
                # the previous drain; block only if nothing has completed
                if d.drain_raw(wait_ms=0) == 0:
                    d.drain_raw(wait_ms=-1)
    while d.pending():
        d.drain_raw(wait_ms=-1)


def stat_delta(a, b):
    return {k: b[k] - a[k] for k in a if isinstance(a[k], (int, float))}


def cpu_baseline(data, off, seconds_budget=12.0):
    """The oracle as it stands, 1 host thread, on a bounded prefix sample."""
    import oracle
    t_total, nbytes, items = 0.0, 0, 0
    st = oracle.Stream()
    k = 0
    n = len(off) - 1
    while k < n and t_total < seconds_budget:
        it = data[int(off[k]):int(off[k + 1])]
        t0 = time.perf_counter()
        st.item(k, it)
        t_total += time.perf_counter() - t0
        nbytes += len(it)
        items += 1
        k += 1
    c = st.counts()
    st.close()
    return {"value": nbytes / t_total / 1e9, "unit": "GB/s", "cores": 1, "kind": "oracle",
            "sample": f"first {items} items ({nbytes / MiB:.0f} MiB) of the {WORKLOAD} stream, "
                      f"sequential C++ oracle (chunk+SHA-1+dedup), {c['chunks']} chunks",
            "chunks_per_s": c["chunks"] / t_total}


def reference_arm(args, data, off):
    """--impl reference: the oracle on the host cores, same metric/config."""
    import oracle
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    n = len(off) - 1
    total_steps = args.steps + args.warmup
    budget_bytes = 60.0 * 60e6       # ~60 s of oracle work (~60 MB/s) over the whole run
    per_step_items = max(1, min(BATCH_ITEMS, int(budget_bytes / max(total_steps, 1) / ITEM_BYTES)))
    st = oracle.Stream()
    k, seq = 0, 0
    t_timed, bytes_timed, chunks_timed = 0.0, 0, 0
    for s in range(total_steps):
        t0 = time.perf_counter()
        nb = nc = 0
        for _ in range(per_step_items):
            if k == n:
                st.close()
                st = oracle.Stream()
                k = 0
            it = data[int(off[k]):int(off[k + 1])]
            r = st.item(seq, it)
            nb += len(it)
            nc += len(r.chunk_start)
            k += 1
            seq += 1
        dt = time.perf_counter() - t0
        if s >= args.warmup:
            t_timed += dt
            bytes_timed += nb
            chunks_timed += nc
    st.close()
    v = bytes_timed / t_timed / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": "GB/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * t_timed / max(args.steps, 1), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "chunks_per_s": chunks_timed / t_timed,
        "config": {"workload": f"{WORKLOAD}: 184 MiB simlarge-sized stream, 1 MiB items, "
                               "dup_frac 0.52", "step_sample_items": per_step_items},
        "cpu_baseline": {"value": v, "unit": "GB/s", "cores": 1, "kind": "oracle",
                         "sample": f"{per_step_items} x 1 MiB items per step, cycling the "
                                   f"{WORKLOAD} stream"},
        "e2e": {"value": v, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


HBM_PEAK = 6462.1  # overwritten from MEASURED_PEAKS.json in main()


def isolated_kernels(dd, off, int_peak, copies=4, reps=3, streams=4):
    """Live per-kernel throughput with the GPU filled by one kernel type.

    chunk stage: one op_chunk call (scan + select) over the C2 stream tiled
    `copies` times (a full-GPU grid).  SHA-1: one launch's duration is floored
    by the longest chunk's serial chain of 64-byte compressions (latency, not
    throughput), so `streams` contexts launch the same SHA-1 work concurrently
    on their own streams and the throughput is all their blocks over the
    joint elapsed time.  CUDA events on torch's current stream bracket both."""
    import torch

    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    nb1 = int(off[-1])
    data = dd.repeat(copies)
    nb = nb1 * copies
    n_items = (len(off) - 1) * copies
    offs = np.concatenate([off[:-1] + k * nb1 for k in range(copies)] + [np.array([nb], off.dtype)])
    item_off = torch.from_numpy(offs.astype(np.int64)).cuda()
    cap = nb // 32 + n_items + 2
    ctxs = [Dedup(0, batch_bytes=nb, batch_items=n_items + 1, slots=1, table_capacity=1 << 12,
                  host_fed=False) for _ in range(streams)]
    try:
        cut = torch.zeros(cap, dtype=torch.int32, device="cuda")
        n = torch.zeros(1, dtype=torch.int32, device="cuda")
        digs = [torch.zeros(cap * 20, dtype=torch.uint8, device="cuda") for _ in range(streams)]
        sts = [torch.cuda.Stream() for _ in range(streams)]
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        ctxs[0].op_chunk(data, nb, item_off, n_items, cut, cap, n)   # warm-up
        ctxs[0].op_sha1(data, nb, cut, n, cap, digs[0])
        torch.cuda.synchronize()
        ev[0].record()
        for _ in range(reps):
            ctxs[0].op_chunk(data, nb, item_off, n_items, cut, cap, n)
        ev[1].record()
        for k in range(streams):
            sts[k].wait_event(ev[1])
            for _ in range(reps):
                ctxs[k].op_sha1(data, nb, cut, n, cap, digs[k], stream=sts[k].cuda_stream)
            torch.cuda.current_stream().wait_stream(sts[k])
        ev[2].record()
        ev[2].synchronize()
        chunk_us = ev[0].elapsed_time(ev[1]) * 1e3 / reps
        sha_us = ev[1].elapsed_time(ev[2]) * 1e3 / (reps * streams)  # per launch's worth
        k = int(n.item())
        cp = cut[:k].cpu().numpy().astype(np.int64)
        # row NEXT-1 (LZSS FindMatch over the same blocks; not part of the step)
        fl = torch.empty(nb, dtype=torch.uint8, device="cuda")
        fo = torch.empty(nb, dtype=torch.int16, device="cuda")
        ctxs[0].op_findmatch(data, nb, cut, n, cap, fl, fo)
        ev[0].record()
        ctxs[0].op_findmatch(data, nb, cut, n, cap, fl, fo)
        ev[1].record()
        ev[1].synchronize()
        fm_us = ev[0].elapsed_time(ev[1]) * 1e3
        # row NEXT-3 (host archive writer) on the first 64 MiB of these outputs
        from paper_conf_ipps_rockenbachsgmtd19_b200 import archive
        an = 64 * MiB
        kk = int(n.item())
        cps = cut[:kk].cpu().numpy().astype(np.int64)
        cps = cps[cps < an].astype(np.uint32)
        a_data = dd[:an].cpu().numpy()
        a_len = fl[:an].cpu().numpy()
        a_off = fo[:an].cpu().numpy().view(np.uint16)
        a_dig = digs[0][:20 * len(cps)].cpu().numpy()
        a_dup = np.zeros(len(cps), np.uint8)
        t0 = time.perf_counter()
        rec = archive.encode(a_data, cps, a_dig, a_dup, a_len, a_off)
        t1 = time.perf_counter()
        back = archive.Decoder().decode(rec, an)
        t2 = time.perf_counter()
        assert np.array_equal(back, a_data)
        arch = {"row": "NEXT-3 (host archive writer: greedy LZSS tokens from FindMatch + "
                       "digest records; C++, 1 host thread)",
                "encode_gbs": an / (t1 - t0) / 1e9, "decode_gbs": an / (t2 - t1) / 1e9,
                "ratio": len(rec) / an, "sample": "first 64 MiB of the C2 stream, every chunk "
                "encoded as unique (the step's duplicates would be 21-byte references)"}
        del fl, fo
    finally:
        for c in ctxs:
            c.close()
    lens = np.diff(np.append(cp, nb))
    blocks = int(((lens + 9 + 63) // 64).sum())
    sha_ops = blocks * SHA1_OPS_PER_BLOCK / (sha_us * 1e-6) / 1e12
    scan_ops = nb * SCAN_OPS_PER_BYTE / (chunk_us * 1e-6) / 1e12
    return {
        "sha1": {"bound": "alu", "achieved": sha_ops, "peak": int_peak, "unit": "Tops/s",
                 "frac": sha_ops / int_peak, "launch_us": sha_us, "launch_bytes": nb,
                 "input_gbs": nb / (sha_us * 1e-6) / 1e9, "blocks": blocks,
                 "note": f"{streams} concurrent streams x {reps} launches; launch_us = "
                         "joint elapsed / launches"},
        "archive": arch,
        "findmatch": {"row": "NEXT-1 (LZSS FindMatch, Listing 3), W=4096, MAX_CODED=18",
                      "bound": "hbm", "achieved": nb * 4 / (fm_us * 1e-6) / 1e9,
                      "peak": HBM_PEAK, "unit": "GB/s",
                      "frac": nb * 4 / (fm_us * 1e-6) / 1e9 / HBM_PEAK,
                      "launch_us": fm_us, "input_gbs": nb / (fm_us * 1e-6) / 1e9,
                      "note": "algorithmic HBM bytes: 1 B read + 3 B written (u8 length, "
                              "u16 offset) per input byte; search-bound, see DESIGN.md"},
        "chunk_stage": {"bound": "alu", "achieved": scan_ops, "peak": int_peak, "unit": "Tops/s",
                        "frac": scan_ops / int_peak, "launch_us": chunk_us,
                        "input_gbs": nb / (chunk_us * 1e-6) / 1e9,
                        "note": "scan + select_scan + select_emit, one op_chunk call; "
                                "HBM: reads 1 B/B -> "
                                f"{nb / (chunk_us * 1e-6) / 1e9 / HBM_PEAK:.3f} of the copy peak"},
    }


# Row NEXT-4 (Mandelbrot Streaming, Section IV-A): the paper's image.
MANDEL_DIM, MANDEL_NITER = 2000, 200000
MANDEL_BATCH_ROWS, MANDEL_SPACES = 1000, 2
# binary64 pipe operations per iteration of Listing 1 (lines 15-19, no FMA):
# a*a, b*b, a2+b2, 2*a, (2a)*b, +im, a2-b2, +cr and the compare with 4.0 (DSETP
# issues to the FP64 pipe: ncu's fp64-pipe utilisation of the kernel matches
# 9 ops x 64 lanes/clk/SM)
MANDEL_FP64_OPS_PER_ITER = 9
# FP64 lanes per SM per clock on B200 (derived: no FP64 figure in
# MEASURED_PEAKS.json / B200_PROFILING.md; 64/clk/SM = the B200 FP64 rating
# of ~37 TFLOPS FMA at 1.965 GHz; ncu's fp64-pipe utilisation checks it)
FP64_LANES_PER_SM_CLK = 64


def mandel_measure(sm_mhz, with_cpu=True):
    from paper_conf_ipps_rockenbachsgmtd19_b200 import mandel as M
    M.image(200, 1000, 32, 2)  # warm-up
    best = None
    for _ in range(3):
        _, ms, iters = M.image(MANDEL_DIM, MANDEL_NITER, MANDEL_BATCH_ROWS, MANDEL_SPACES)
        best = ms if best is None else min(best, ms)
    peak = 148 * FP64_LANES_PER_SM_CLK * sm_mhz * 1e6 / 1e12
    ach = iters * MANDEL_FP64_OPS_PER_ITER / (best * 1e-3) / 1e12
    out = {"row": "NEXT-4 (Mandelbrot Streaming, Listings 1-2)",
           "workload": f"{MANDEL_DIM}x{MANDEL_DIM}, niter {MANDEL_NITER} (P:131), frame "
                       f"[-2.125, 0.875] x [-1.5, 1.5], batches of {MANDEL_BATCH_ROWS} rows, "
                       f"{MANDEL_SPACES} memory spaces, D2H into pinned host memory",
           "image_ms": best, "iterations": iters, "t_iter_per_s": iters / (best * 1e-3) / 1e12,
           "bound": "fp64", "achieved": ach, "peak": peak, "unit": "T binary64 pipe ops/s",
           "frac": ach / peak,
           "peak_source": f"derived: 148 SM x {FP64_LANES_PER_SM_CLK} FP64 lanes/clk x "
                          f"{sm_mhz:.0f} MHz",
           "paper_context": "400 s sequential (i9-7900X), 3.02 s on 2x Titan XP (P:131, P:185)"}
    if with_cpu:
        import oracle
        t0 = time.perf_counter()
        oracle.mandel_rows(MANDEL_DIM, MANDEL_NITER, row0=1000, nrows=1)
        dt = time.perf_counter() - t0
        step = 3.0 / MANDEL_DIM
        row_iters = sum(oracle.mandel_iters(-2.125 + step * j, -1.5 + step * 1000, MANDEL_NITER)
                        for j in range(MANDEL_DIM))
        out["cpu_baseline"] = {"value": row_iters / dt / 1e12, "unit": "T iter/s", "cores": 1,
                               "kind": "oracle", "sample": "row 1000 (the densest) of the image"}
    return out


def batch_sweep(dd, off, sizes=(1, 2, 4, 8, 16, 32), target_bytes=3 << 30):
    """BASELINE.json configs[1]: the C2 stream at GPU batch sizes 1..32 MiB
    (the 64 MiB point is the headline `value`), device-resident, 40 batches
    in flight, CUDA events around the submissions; GB/s per batch size."""
    import torch

    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    out = {}
    for mb in sizes:
        bb = mb * MiB
        plan, k, n = [], 0, len(off) - 1
        while k < n:
            j = k + 1
            while j < n and int(off[j + 1]) - int(off[k]) <= bb:
                j += 1
            plan.append((k, j))
            k = j
        subs = [(dd[int(off[a]):int(off[b])], (off[a:b + 1] - off[a]).copy()) for a, b in plan]
        d = Dedup(0, batch_bytes=bb, batch_items=max(mb, 1) + 1, slots=SLOTS,
                  table_capacity=max(1 << 16, len(dd) // 2048), host_fed=False)
        producer = torch.cuda.current_stream().cuda_stream
        sub = lambda b: d.submit_device(subs[b][0], subs[b][1], producer)  # noqa: E731
        steps = max(400, target_bytes // bb)
        run_steps(d, sub, len(plan), 8, 0)
        torch.cuda.synchronize()
        s0 = d.stats()
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
        ev[0].record()
        run_steps(d, sub, len(plan), steps, 8)
        d.join()
        ev[1].record()
        ev[1].synchronize()
        nbytes = d.stats()["bytes"] - s0["bytes"]
        out[f"{mb}MiB"] = nbytes / (ev[0].elapsed_time(ev[1]) * 1e-3) / 1e9
        d.close()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=600)
    ap.add_argument("--warmup", type=int, default=12)
    ap.add_argument("--impl", default="b200", choices=["b200", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=0, help="0 = min(steps, 120)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--batch-mb", type=int, default=0, help="override the GPU batch size")
    ap.add_argument("--slots", type=int, default=0, help="override the in-flight batches")
    ap.add_argument("--step-only", action="store_true",
                    help="time the step only (no isolated-kernel, NEXT-row, e2e or CPU legs): "
                         "for the ncu launch list of the step")
    args = ap.parse_args()
    global BATCH_BYTES, SLOTS, BATCH_ITEMS
    if args.batch_mb:
        BATCH_BYTES = args.batch_mb * MiB
        BATCH_ITEMS = max(BATCH_ITEMS, BATCH_BYTES // ITEM_BYTES)
    if args.slots:
        SLOTS = args.slots
    if args.warmup < 3:
        args.warmup = 3

    data = synthgen.config_stream(WORKLOAD)
    off = synthgen.split_items(data, ITEM_BYTES)

    if args.impl == "reference":
        return reference_arm(args, data, off)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world > 1 or args.gpus > 1:
        from paper_conf_ipps_rockenbachsgmtd19_b200 import dist_bench
        # pass this module: under torchrun bench.py runs as __main__, and an
        # `import bench` would see the default (un-overridden) batch settings
        return dist_bench.main(args, data, off, sys.modules[__name__])

    import torch

    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup

    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    plan = plan_batches(off)
    nb = len(plan)
    dd = torch.from_numpy(data).to(dev)
    subs = []
    for k, j in plan:
        subs.append((dd[int(off[k]):int(off[j])], (off[k:j + 1] - off[k]).copy()))
    batch_bytes = [int(off[j]) - int(off[k]) for k, j in plan]

    d = Dedup(0, **engine_kwargs(len(data)))
    producer = torch.cuda.current_stream().cuda_stream
    submit_dev = lambda b: d.submit_device(subs[b][0], subs[b][1], producer)  # noqa: E731
    torch.cuda.synchronize()

    # ---- device-resident (value) ----
    run_steps(d, submit_dev, nb, args.warmup, 0)
    torch.cuda.synchronize()
    s0 = d.stats()
    l0 = d.kernel_launches()
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(0) as clk:
        start.record()
        run_steps(d, submit_dev, nb, args.steps, args.warmup)
        d.join()
        end.record()
        end.synchronize()
    ms = start.elapsed_time(end)
    s1 = d.stats()
    launches = d.kernel_launches() - l0
    ds = stat_delta(s0, s1)
    step_ids = [(args.warmup + s) % nb for s in range(args.steps)]
    bytes_timed = sum(batch_bytes[b] for b in step_ids)
    assert ds["bytes"] == bytes_timed, (ds["bytes"], bytes_timed)
    value = bytes_timed / (ms / 1e3) / 1e9
    chunks_per_s = ds["chunks"] / (ms / 1e3)

    # ---- rooflines ----
    pk, src = peaks()
    global HBM_PEAK
    HBM_PEAK = float(pk.get("hbm_gbs", HBM_PEAK))
    clocks = clk.summary()
    sm_mhz = pk.get("sm_max_mhz", 1965.0)
    int_peak = 148 * INT_LANES_PER_SM_CLK * sm_mhz * 1e6 / 1e12      # Tops/s
    peak_source = (f"derived: 148 SM x 4 SMSP x 32 lanes (1 warp-instr/clk/SMSP) x "
                   f"{sm_mhz:.0f} MHz ({src} max SM clock); B200_PROFILING.md has no "
                   "integer peak")
    # pipeline stage latencies: CUDA events of every DEDUP_TIME_EVERY-th batch on
    # the slot's own stream (the stages of ~SLOTS batches overlap, so these are
    # latencies, not costs)
    nt = max(ds["timed_batches"], 1)
    kernels = {
        "stage_latency_ms_per_batch": {
            "rabin_scan": ds["ms_scan"] / nt, "select+meta": ds["ms_select"] / nt,
            "sha1": ds["ms_sha1"] / nt, "table": ds["ms_table"] / nt,
            "pack_d2h": ds["ms_d2h"] / nt},
        "timed_batches": ds["timed_batches"],
    }
    if args.step_only:
        print(json.dumps({"metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": 1,
                          "steps": args.steps, "warmup": args.warmup,
                          "ms_per_step": ms / args.steps, "gpu_launches": launches,
                          "note": "--step-only"}), flush=True)
        d.close()
        return
    iso = isolated_kernels(dd, off, int_peak)
    kernels.update(iso)
    kernels["mandelbrot"] = mandel_measure(sm_mhz, with_cpu=not args.no_cpu_baseline)
    sweep = batch_sweep(dd, off)
    sweep[f"{BATCH_BYTES // MiB}MiB"] = value
    sha_blocks_per_byte = ds["sha1_blocks"] / max(ds["bytes"], 1)
    path_ops = value * 1e9 * (SCAN_OPS_PER_BYTE + sha_blocks_per_byte * SHA1_OPS_PER_BLOCK) / 1e12
    kernels["path"] = {"bound": "alu", "achieved": path_ops, "peak": int_peak, "unit": "Tops/s",
                       "frac": path_ops / int_peak,
                       "ops_per_byte": SCAN_OPS_PER_BYTE + sha_blocks_per_byte * SHA1_OPS_PER_BLOCK,
                       "note": "whole step: algorithmic scan + SHA-1 int ops at `value`"}
    # dominant kernel: SHA-1 (largest marginal cost per batch in the pipeline,
    # DESIGN.md section 8); achieved = its algorithmic ops per launch / launch
    # duration of an isolated full-GPU launch on the C2 data
    kd = kernels["sha1"]
    traffic = None
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp):  # DRAM bytes per launch from the committed ncu capture,
        tj = json.load(open(tp))  # scaled from its batch size to this launch's bytes
        if "sha1" in tj:
            traffic = tj["sha1"] / tj["capture_batch_bytes"] * kd["launch_bytes"]
    # the same launch against the ALU pipe alone (16 lanes/clk/SMSP): the
    # round function and message schedule need 432 ALU-pipe ops per block
    # (f LOP3 80, rotl30 SHF 80, rotl5+add LEA 80, schedule 2 LOP3 + SHF
    # per word x 64), the adds go to the FMA pipe
    alu_peak = int_peak / 2
    alu_ach = kd["achieved"] * SHA1_ALU_OPS_PER_BLOCK / SHA1_OPS_PER_BLOCK
    roofline = {"kernel": "sha1_kernel", "bound": "alu", "achieved": kd["achieved"],
                "peak": int_peak, "unit": "Tops/s", "frac": kd["achieved"] / int_peak,
                "alu_pipe_view": {"achieved": alu_ach, "peak": alu_peak,
                                  "frac": alu_ach / alu_peak, "ops_per_block":
                                  SHA1_ALU_OPS_PER_BLOCK},
                "traffic": traffic, "peak_source": peak_source,
                "launch": f"{kd['launch_bytes'] / MiB:.0f} MiB of C2 chunks per launch, "
                          f"{kd['launch_us']:.0f} us per launch (CUDA events, "
                          "4 concurrent streams)"}

    # ---- end-to-end through the host-fed C ABI ----
    e2e_steps = args.e2e_steps or min(args.steps, 120)
    pin = d.host_empty(len(data))
    pin[:] = data
    submit_host = lambda b: d.submit_buffer(  # noqa: E731
        pin[int(off[plan[b][0]]):int(off[plan[b][1]])], subs[b][1])
    d.end_stream()
    run_steps(d, submit_host, nb, args.warmup, 0)
    torch.cuda.synchronize()
    e0 = d.stats()
    start.record()
    run_steps(d, submit_host, nb, e2e_steps, args.warmup)
    d.join()
    end.record()
    end.synchronize()
    ems = start.elapsed_time(end)
    e1 = d.stats()
    de = stat_delta(e0, e1)
    e2e_value = de["bytes"] / (ems / 1e3) / 1e9
    items_per_step = de["items"] / e2e_steps
    e2e = {"value": e2e_value, "unit": "GB/s",
           "h2d_bytes_per_step": (de["bytes"] + 8 * (de["items"] + de["batches"])) / e2e_steps,
           "d2h_bytes_per_step": (33 * de["chunks"] + 4 * de["items"] + 8 * de["batches"])
           / e2e_steps,
           "steps": e2e_steps, "items_per_step": items_per_step,
           "api": "dedup_submit_batch (pinned host buffers) + dedup_drain",
           "pcie_h2d_gbs": h2d_bandwidth(pin, dd)}
    d.close()

    line = {
        "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "chunks_per_s": chunks_per_s,
        "dup_ratio": ds["dup_chunks"] / max(ds["chunks"], 1),
        "config": {"workload": f"{WORKLOAD}: 184 MiB simlarge-sized synthetic stream (seed 2), "
                               "1 MiB items, dup_frac 0.52, device-resident",
                   "batch_bytes": BATCH_BYTES, "batch_items": BATCH_ITEMS, "slots": SLOTS,
                   "batches_per_stream": nb, "parallelism": "1 GPU",
                   "batch_sweep_gbs": sweep,
                   "l2": "inputs larger than L2 (184 MiB stream cycled, 126 MB L2)"},
        "clocks": clocks, "gpu_launches": launches, "roofline": roofline, "kernels": kernels,
        "e2e": e2e,
    }
    if not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(data, off)
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
