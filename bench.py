#!/usr/bin/env python
"""Benchmark of the GPU Dedup hot path (Rabin CDC -> SHA-1 -> global dedup).

Contract (README / DESIGN.md "Measurement"):
  python bench.py --gpus N --steps K --warmup W [--impl b200|reference]
prints ONE JSON line on rank 0.

Workload: BASELINE.json configs[2], the 672 MiB native-sized synthetic stream
C3 (1 MiB items, dup_frac 0.52), resident in HBM.  A step is one pass of the
whole hot path (rows A1-A9 of SURVEY 8(a)) over the WHOLE C3 stream as a new
dedup stream (fresh digest table): 11 GPU batches (64 MiB of whole items
each).  The engine keeps up to SLOTS batches in flight and consecutive steps
run back to back (a step's batches enter the pipeline while the previous
step's are still in flight), so the timed region -- W warm-up steps drained,
then K steps bracketed by CUDA events -- measures the pipeline in steady
state plus one fill and one drain.  `value` is input GB/s (1e9 B/s); `e2e`
is the same metric through dedup_submit_batch with pinned HOST buffers (H2D
and the result read-back inside the timed region).
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
# host time)
os.environ.setdefault("DEDUP_TIME_EVERY", "8")

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import synthgen  # noqa: E402

MiB = 1 << 20
ITEM_BYTES = MiB                 # the paper's fixed 1 MB batches
BATCH_BYTES = 64 * MiB           # GPU batch; configs[1] sweeps 1-64 MiB
BATCH_ITEMS = 64
SLOTS = 40                       # batches in flight ("memory spaces")
WORKLOAD = "C3"
WORKLOAD_DESC = ("C3: 672 MiB native-sized synthetic stream (seed 3), 1 MiB items, "
                 "dup_frac 0.52, device-resident; one step = one pass over the whole stream "
                 "as a new dedup stream (11 GPU batches of <= 64 MiB)")
METRIC = "input GB/s & chunks/s (dedup hot path) at 1/2/4/8 B200; % of HBM/INT roofline"

# SHA-1 algorithmic 32-bit integer ops per 64-byte block (FIPS 180-4 6.1.2,
# counting a 3-input logic/add as one op and a rotate as one op):
#   80 rounds x (f 1 + rotl5 1 + adds 2 + rotl30 1) + 64 x schedule 3 + 5.
SHA1_OPS_PER_BLOCK = 80 * 5 + 64 * 3 + 5
# of which, as the minimal sm_100a mapping issues them:
# on the ALU pipe f LOP3 80, rotl30 SHF 80, rotl5 + add LEA.HI 80, schedule
# 2 LOP3 + 1 SHF per word x 64 = 432; on the FMA pipe the other adds 165
SHA1_ALU_OPS_PER_BLOCK = 80 * 3 + 64 * 3
SHA1_FMA_OPS_PER_BLOCK = SHA1_OPS_PER_BLOCK - SHA1_ALU_OPS_PER_BLOCK
# Rabin rolling step per input byte: 2 table lookups, shift-in,
# 2 address formations, 1 3-way XOR, test + bit = 8 ops.
SCAN_OPS_PER_BYTE = 8


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        return json.load(open(p)), "measured"
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
            time.sleep(0.002)

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


def plan_batches(off, batch_bytes=None, batch_items=None):
    """Greedy grouping of whole items into GPU batches (item index ranges)."""
    bb = batch_bytes or BATCH_BYTES
    bi = batch_items or BATCH_ITEMS
    out, k, n = [], 0, len(off) - 1
    while k < n:
        j = k + 1
        while j < n and j - k < bi and int(off[j + 1]) - int(off[k]) <= bb:
            j += 1
        out.append((k, j))
        k = j
    return out


SHA_LANE = 0                     # batch bytes per SHA-1 lane (0: the engine's 16 KiB)


def engine_kwargs(stream_bytes: int) -> dict:
    return dict(batch_bytes=BATCH_BYTES, batch_items=BATCH_ITEMS, slots=SLOTS,
                table_capacity=max(1 << 16, stream_bytes // 2048), host_fed=True,
                sha_lane_bytes=SHA_LANE)


def submit_pass(d, submit, n_batches, new_stream=True):
    """One step: every batch of the stream, as a new dedup stream.  A full
    slot ring is relieved by a non-blocking drain (results of the batches
    handed out by the previous drain are released), blocking only if nothing
    has completed."""
    if new_stream:  # (carry-over mode: may need a slot for the closing item)
        while True:
            try:
                d.end_stream()
                break
            except Exception as e:
                if "EAGAIN" not in str(e):
                    raise
                if d.drain_raw(wait_ms=0) == 0:
                    d.drain_raw(wait_ms=-1)
    for b in range(n_batches):
        while True:
            try:
                submit(b)
                break
            except Exception as e:
                if "EAGAIN" not in str(e):
                    raise
                if d.drain_raw(wait_ms=0) == 0:
                    d.drain_raw(wait_ms=-1)


def drain_all(d):
    while d.pending():
        d.drain_raw(wait_ms=-1)


def stat_delta(a, b):
    return {k: b[k] - a[k] for k in a if isinstance(a[k], (int, float))}


def timed_passes(d, submit, n_batches, steps, warmup, sampler=None):
    """W warm-up passes (drained), then K passes between CUDA events on
    torch's stream; dedup_join makes the end event wait for every batch."""
    import torch
    for _ in range(warmup):
        submit_pass(d, submit, n_batches)
    drain_all(d)
    torch.cuda.synchronize()
    s0, l0 = d.stats(), d.kernel_launches()
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ctx = sampler if sampler is not None else _Null()
    with ctx:
        start.record()
        for _ in range(steps):
            submit_pass(d, submit, n_batches)
        d.join()
        end.record()
        end.synchronize()
    drain_all(d)
    ms = start.elapsed_time(end)
    return ms, stat_delta(s0, d.stats()), d.kernel_launches() - l0


class _Null:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        return False


def device_subs(dd, off, plan):
    return [(dd[int(off[k]):int(off[j])], (off[k:j + 1] - off[k]).copy()) for k, j in plan]


def stream_throughput(name, data, steps=3, warmup=1, distinct=None):
    """GB/s and chunks/s of the engine on one named config (device-resident,
    the bench's engine configuration, each pass a new dedup stream).
    distinct: expected distinct chunks per pass (digest-table capacity)."""
    import torch

    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    off = synthgen.split_items(data, ITEM_BYTES)
    plan = plan_batches(off)
    dd = torch.from_numpy(data).cuda()
    subs = device_subs(dd, off, plan)
    kw = dict(engine_kwargs(len(data)), host_fed=False)
    if distinct:
        kw["table_capacity"] = max(kw["table_capacity"], distinct)
    with Dedup(0, **kw) as d:
        prod = torch.cuda.current_stream().cuda_stream
        ms, ds, _ = timed_passes(d, lambda b: d.submit_device(subs[b][0], subs[b][1], prod),
                                 len(plan), steps, warmup)
    del dd, subs
    torch.cuda.empty_cache()
    return {"gbs": ds["bytes"] / (ms * 1e-3) / 1e9, "chunks_per_s": ds["chunks"] / (ms * 1e-3),
            "chunks_per_pass": ds["chunks"] // steps,
            "dup_ratio": ds["dup_chunks"] / max(ds["chunks"], 1),
            "bytes_per_pass": ds["bytes"] // steps, "passes": steps}


def carry_throughput(data, piece=61 * MiB + 48, steps=4, warmup=1):
    """Row NEXT-2, carry-over mode: the stream as ONE chunking domain cut into
    pieces of `piece` bytes (not item- or chunk-aligned), device-resident,
    one piece per batch, each pass a new dedup stream closed by end_stream."""
    import torch

    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    dd = torch.from_numpy(data).cuda()
    bounds = [(a, min(a + piece, len(data))) for a in range(0, len(data), piece)]
    subs = [(dd[a:b], np.array([0, b - a], np.uint64)) for a, b in bounds]
    with Dedup(0, batch_bytes=piece, batch_items=1, slots=SLOTS, carry_over=True,
               table_capacity=max(1 << 16, len(data) // 2048), host_fed=False) as d:
        prod = torch.cuda.current_stream().cuda_stream

        def submit(b):
            d.submit_device(subs[b][0], subs[b][1], prod)

        ms, ds, _ = timed_passes(d, submit, len(subs), steps, warmup)
    del dd, subs
    torch.cuda.empty_cache()
    return {"gbs": ds["bytes"] / (ms * 1e-3) / 1e9, "chunks_per_s": ds["chunks"] / (ms * 1e-3),
            "chunks_per_pass": ds["chunks"] // steps, "piece_bytes": piece, "passes": steps,
            "workload": "C3 as one chunking domain (carry-over mode, row NEXT-2), cut into "
                        f"{len(bounds)} pieces of {piece} B, one piece per batch"}


def config_lines(steps):
    """Throughput of the other BASELINE.json configs (single GPU)."""
    out = {}
    specs = [
        ("C1", "10 MiB simsmall-sized, dup_frac 0.52 (seed 1)", lambda: synthgen.config_stream("C1")),
        ("C4_share", "the 2 GiB per-GPU share (1/8) of the 16 GiB dup_frac-0 stream (seed 4)",
         lambda: synthgen.config_stream("C4", nbytes=2 << 30)),
        ("C5a", "672 MiB all-unique (seed 51)", lambda: synthgen.config_stream("C5a")),
        ("C5b", "672 MiB all-duplicate: every item = item 0 (seed 52)",
         lambda: synthgen.config_stream("C5b")),
        ("C5c_zero", "672 MiB all-zero: 22 M identical 32-byte chunks",
         lambda: synthgen.config_stream("C5c_zero")),
        ("C5c_hit", "672 MiB constructed-hit: 22 M distinct 32-byte chunks",
         lambda: synthgen.config_stream("C5c_hit")),
        ("C5d", "672 MiB constructed no-hit: one 1 MiB chunk per item",
         lambda: synthgen.config_stream("C5d")),
    ]
    for key, desc, gen in specs:
        data = gen()
        # about 0.3-3 GB of work per config: C1 is tiny, repeat it more
        n = max(1, min(steps, int(3e9 // len(data))))
        try:
            r = stream_throughput(key, data, steps=n,
                                  distinct=len(data) // 32 + 1 if key == "C5c_hit" else None)
        except Exception as e:  # report, keep the bench line
            r = {"error": str(e)[:200]}
        r["workload"] = desc
        out[key] = r
        del data
    return out


def batch_sweep(data, sizes=(1, 2, 4, 8, 16, 32, 64), target_bytes=2 << 30):
    """BASELINE.json configs[1]: the C2 stream at GPU batch sizes 1..64 MiB,
    device-resident, SLOTS batches in flight; GB/s per batch size."""
    import torch

    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    out = {}
    off = synthgen.split_items(data, ITEM_BYTES)
    dd = torch.from_numpy(data).cuda()
    for mb in sizes:
        bb = mb * MiB
        plan = plan_batches(off, bb, max(mb, 1) + 1)
        subs = device_subs(dd, off, plan)
        with Dedup(0, batch_bytes=bb, batch_items=max(mb, 1) + 1, slots=SLOTS,
                   table_capacity=max(1 << 16, len(data) // 2048), host_fed=False) as d:
            prod = torch.cuda.current_stream().cuda_stream
            # enough batches that the SLOTS in flight reach steady state
            passes = max(2, int(max(target_bytes, 4 * SLOTS * bb) // len(data)))
            ms, ds, _ = timed_passes(
                d, lambda b: d.submit_device(subs[b][0], subs[b][1], prod), len(plan),
                passes, 1)
        out[f"{mb}MiB"] = ds["bytes"] / (ms * 1e-3) / 1e9
    del dd
    torch.cuda.empty_cache()
    return out


def int_rates():
    """Measured integer-pipe rates (include/dedup.h dedup_probe_int_rates)."""
    from paper_conf_ipps_rockenbachsgmtd19_b200 import probe_int_rates
    return probe_int_rates(0)


def sha1_peak(r):
    """Attainable int ops/s for SHA-1's op mix from the measured pipe rates:
    a block needs 432 ALU-pipe ops, 165 FMA-pipe ops and 597 issue slots, so
    its time is max(432 / R_alu, 165 / R_fma, 597 / R_issue)."""
    t = max(SHA1_ALU_OPS_PER_BLOCK / r["lop3"], SHA1_FMA_OPS_PER_BLOCK / r["imad"],
            SHA1_OPS_PER_BLOCK / r["mix_lop3_imad"])
    return SHA1_OPS_PER_BLOCK / t


def isolated_kernels(dd, off, int_peak, alu_peak, reps=3, streams=12):
    """Live per-kernel throughput with the GPU filled by one kernel type, on
    the C3 stream.  chunk stage: one op_chunk call (scan + cut selection)
    over the whole stream.  SHA-1: one launch's duration is floored by its
    longest chunk's serial chain of 64-byte compressions (latency, not
    throughput), so `streams` contexts launch the same SHA-1 work
    concurrently on their own streams and the throughput is all their blocks
    over the joint elapsed time.  12 concurrent launches keep every SM's 4
    SHA-1 CTA slots busy through each launch's tail (measured with 32 KiB
    lanes, 84 CTAs per launch: 4 / 8 / 12 launches 1.64-1.67 / 1.72-1.74 /
    1.82-1.85 TB/s; 8 launches of 16 KiB lanes 1.83-1.86).  CUDA events on torch's stream bracket both."""
    import torch

    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    nb = int(off[-1])
    n_items = len(off) - 1
    item_off = torch.from_numpy(off.astype(np.int64)).cuda()
    cap = nb // 32 + n_items + 2
    ctxs = [Dedup(0, batch_bytes=nb, batch_items=n_items + 1, slots=1, table_capacity=1 << 12,
                  host_fed=False) for _ in range(streams)]
    try:
        cut = torch.zeros(cap, dtype=torch.int32, device="cuda")
        n = torch.zeros(1, dtype=torch.int32, device="cuda")
        digs = [torch.zeros(cap * 20, dtype=torch.uint8, device="cuda") for _ in range(streams)]
        sts = [torch.cuda.Stream() for _ in range(streams)]
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        ctxs[0].op_chunk(dd, nb, item_off, n_items, cut, cap, n)   # warm-up
        ctxs[0].op_sha1(dd, nb, cut, n, cap, digs[0])
        torch.cuda.synchronize()
        ev[0].record()
        for _ in range(reps):
            ctxs[0].op_chunk(dd, nb, item_off, n_items, cut, cap, n)
        ev[1].record()
        for k in range(streams):
            sts[k].wait_event(ev[1])
            for _ in range(reps):
                ctxs[k].op_sha1(dd, nb, cut, n, cap, digs[k], stream=sts[k].cuda_stream)
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
        ctxs[0].op_findmatch(dd, nb, cut, n, cap, fl, fo)
        ev[0].record()
        ctxs[0].op_findmatch(dd, nb, cut, n, cap, fl, fo)
        ev[1].record()
        ev[1].synchronize()
        fm_us = ev[0].elapsed_time(ev[1]) * 1e3
        # row NEXT-3 (host archive writer) on the first 64 MiB of these outputs
        from paper_conf_ipps_rockenbachsgmtd19_b200 import archive
        an = 64 * MiB
        cps = cp[cp < an].astype(np.uint32)
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
                "ratio": len(rec) / an, "sample": "first 64 MiB of the C3 stream, every chunk "
                "encoded as unique (the step's duplicates would be 21-byte references)"}
        del fl, fo
    finally:
        for c in ctxs:
            c.close()
    lens = np.diff(np.append(cp, nb))
    blocks = int(((lens + 9 + 63) // 64).sum())
    sha_ops = blocks * SHA1_OPS_PER_BLOCK / (sha_us * 1e-6) / 1e12
    scan_ops = nb * SCAN_OPS_PER_BYTE / (chunk_us * 1e-6) / 1e12
    pk, _ = peaks()
    hbm = float(pk.get("hbm_gbs", 6550.1))
    return {
        "sha1": {"bound": "alu", "achieved": sha_ops, "peak": int_peak, "unit": "Tops/s",
                 "frac": sha_ops / int_peak, "launch_us": sha_us, "launch_bytes": nb,
                 "input_gbs": nb / (sha_us * 1e-6) / 1e9, "blocks": blocks,
                 "note": f"{streams} concurrent streams x {reps} launches over the C3 chunks; "
                         "launch_us = joint elapsed / launches"},
        "archive": arch,
        "findmatch": {"row": "NEXT-1 (LZSS FindMatch, Listing 3), W=4096, MAX_CODED=18",
                      "bound": "hbm", "achieved": nb * 4 / (fm_us * 1e-6) / 1e9,
                      "peak": hbm, "unit": "GB/s",
                      "frac": nb * 4 / (fm_us * 1e-6) / 1e9 / hbm,
                      "launch_us": fm_us, "input_gbs": nb / (fm_us * 1e-6) / 1e9,
                      "note": "algorithmic HBM bytes: 1 B read + 3 B written (u8 length, "
                              "u16 offset) per input byte; search-bound, see DESIGN.md"},
        "chunk_stage": {"bound": "alu", "achieved": scan_ops, "peak": alu_peak, "unit": "Tops/s",
                        "frac": scan_ops / alu_peak, "launch_us": chunk_us,
                        "input_gbs": nb / (chunk_us * 1e-6) / 1e9,
                        "hbm_frac": nb / (chunk_us * 1e-6) / 1e9 / hbm,
                        "note": "scan + select_scan + select_emit, one op_chunk call over C3; "
                                "peak = measured LOP3 (ALU-pipe) rate; hbm_frac = read "
                                "bytes / the HBM copy peak"},
    }


# Row NEXT-4 (Mandelbrot Streaming, Section IV-A): the paper's image.
MANDEL_DIM, MANDEL_NITER = 2000, 200000
MANDEL_BATCH_ROWS, MANDEL_SPACES = 1000, 2
# binary64 pipe operations per iteration of Listing 1 (lines 15-19, no FMA):
# a*a, b*b, a2+b2, 2*a, (2a)*b, +im, a2-b2, +cr and the compare with 4.0
MANDEL_FP64_OPS_PER_ITER = 9
# FP64 lanes per SM per clock on B200 (derived: no FP64 figure in
# MEASURED_PEAKS.json / B200_PROFILING.md; ncu's fp64-pipe utilisation checks it)
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


def host_info():
    info = {"nproc": os.cpu_count()}
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                info["cpu"] = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return info


def cpu_baseline(data, off, seconds_budget=12.0):
    """The oracle as it stands on the host cores, on a bounded prefix of the
    stream: (1) the threaded driver (chunking + SHA-1 of the items on all
    cores, the dedup table sequential) and (2) the
    sequential oracle on one core."""
    import oracle
    T = os.cpu_count() or 1
    n = len(off) - 1
    # calibrate the threaded driver on a few items, then size the sample
    k0 = min(n, max(4, T))
    st = oracle.Stream()
    t0 = time.perf_counter()
    st.items_parallel(0, data[:int(off[k0])], off[:k0 + 1], T)
    rate = int(off[k0]) / (time.perf_counter() - t0)
    st.close()
    k = int(min(n, max(k0, rate * seconds_budget * 0.6 // ITEM_BYTES)))
    st = oracle.Stream()
    t0 = time.perf_counter()
    r = st.items_parallel(0, data[:int(off[k])], off[:k + 1], T)
    dt = time.perf_counter() - t0
    st.close()
    nbytes = int(off[k])
    out = {"value": nbytes / dt / 1e9, "unit": "GB/s", "cores": T, "kind": "oracle",
           "sample": f"first {k} items ({nbytes / MiB:.0f} MiB) of the {WORKLOAD} stream, "
                     f"threaded oracle driver: chunking + SHA-1 on {T} threads "
                     f"({r.s_chunk_sha:.2f} s), dedup table sequential ({r.s_dedup:.3f} s)",
           "chunks_per_s": len(r.chunk_start) / dt, "host": host_info()}
    # one core, the sequential oracle (about a third of the budget)
    st = oracle.Stream()
    t1, nb1, j = 0.0, 0, 0
    while j < n and t1 < seconds_budget * 0.3:
        it = data[int(off[j]):int(off[j + 1])]
        t0 = time.perf_counter()
        st.item(j, it)
        t1 += time.perf_counter() - t0
        nb1 += len(it)
        j += 1
    st.close()
    out["one_core"] = {"value": nb1 / t1 / 1e9, "unit": "GB/s", "cores": 1,
                       "sample": f"first {j} items, sequential oracle"}
    return out


def reference_arm(args, data, off):
    """--impl reference: the oracle on the host cores, same metric/config.
    Each step is a bounded sample of the C3 stream (its first items, one new
    dedup stream per step) through the threaded oracle driver on all cores,
    sized from a calibration so the whole run takes about a minute."""
    import oracle
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    T = os.cpu_count() or 1
    n = len(off) - 1
    total_steps = args.steps + args.warmup
    k0 = min(n, max(4, T))
    st = oracle.Stream()
    t0 = time.perf_counter()
    st.items_parallel(0, data[:int(off[k0])], off[:k0 + 1], T)
    rate = int(off[k0]) / (time.perf_counter() - t0)
    st.close()
    per_step = int(min(n, max(k0, rate * 60.0 / max(total_steps, 1) // ITEM_BYTES)))
    t_timed, bytes_timed, chunks_timed = 0.0, 0, 0
    for s in range(total_steps):
        st = oracle.Stream()
        t0 = time.perf_counter()
        r = st.items_parallel(0, data[:int(off[per_step])], off[:per_step + 1], T)
        dt = time.perf_counter() - t0
        st.close()
        if s >= args.warmup:
            t_timed += dt
            bytes_timed += int(off[per_step])
            chunks_timed += len(r.chunk_start)
    v = bytes_timed / t_timed / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": "GB/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * t_timed / max(args.steps, 1), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "chunks_per_s": chunks_timed / t_timed,
        "config": {"workload": WORKLOAD_DESC, "step_sample_items": per_step},
        "cpu_baseline": {"value": v, "unit": "GB/s", "cores": T, "kind": "oracle",
                         "sample": f"first {per_step} x 1 MiB items of the {WORKLOAD} stream "
                                   "per step (a new dedup stream each step), threaded oracle "
                                   f"driver on {T} threads", "host": host_info()},
        "e2e": {"value": v, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="b200", choices=["b200", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=0, help="0 = steps")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--slots", type=int, default=0, help="override the in-flight batches")
    ap.add_argument("--sha-lane", type=int, default=0,
                    help="override the batch bytes per SHA-1 lane (0 = the engine default)")
    ap.add_argument("--step-only", action="store_true",
                    help="time the step only (no isolated-kernel, config, NEXT-row, e2e or CPU "
                         "legs): for the ncu launch list of the step")
    args = ap.parse_args()
    global SLOTS, SHA_LANE
    if args.slots:
        SLOTS = args.slots
    if args.sha_lane:
        SHA_LANE = args.sha_lane
    if args.warmup < 3:
        args.warmup = 3

    data = synthgen.config_stream(WORKLOAD)
    off = synthgen.split_items(data, ITEM_BYTES)

    if args.impl == "reference":
        return reference_arm(args, data, off)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world > 1 or args.gpus > 1:
        from paper_conf_ipps_rockenbachsgmtd19_b200 import dist_bench
        # pass this module: under torchrun bench.py runs as __main__
        return dist_bench.main(args, data, off, sys.modules[__name__])

    import torch

    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup

    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    plan = plan_batches(off)
    nb = len(plan)
    dd = torch.from_numpy(data).to(dev)
    subs = device_subs(dd, off, plan)
    d = Dedup(0, **engine_kwargs(len(data)))
    producer = torch.cuda.current_stream().cuda_stream
    submit_dev = lambda b: d.submit_device(subs[b][0], subs[b][1], producer)  # noqa: E731
    torch.cuda.synchronize()

    # ---- device-resident (value) ----
    clk = ClockSampler(0)
    ms, ds, launches = timed_passes(d, submit_dev, nb, args.steps, args.warmup, clk)
    bytes_timed = args.steps * int(off[-1])
    assert ds["bytes"] == bytes_timed, (ds["bytes"], bytes_timed)
    value = bytes_timed / (ms / 1e3) / 1e9
    chunks_per_s = ds["chunks"] / (ms / 1e3)
    clocks = clk.summary()
    if args.step_only:
        print(json.dumps({"metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": 1,
                          "steps": args.steps, "warmup": args.warmup,
                          "ms_per_step": ms / args.steps, "gpu_launches": launches,
                          "chunks_per_s": chunks_per_s, "clocks": clocks,
                          "note": "--step-only"}), flush=True)
        d.close()
        return

    # ---- measured roofline denominators ----
    pk, src = peaks()
    hbm_peak = float(pk.get("hbm_gbs", 6550.1))
    sm_mhz = pk.get("sm_max_mhz", 1965.0)
    rates = int_rates()
    int_peak = sha1_peak(rates)
    alu_peak = rates["lop3"]
    nt = max(ds["timed_batches"], 1)
    kernels = {
        "stage_latency_ms_per_batch": {
            "rabin_scan": ds["ms_scan"] / nt, "select+meta": ds["ms_select"] / nt,
            "sha1": ds["ms_sha1"] / nt, "table": ds["ms_table"] / nt,
            "pack_d2h": ds["ms_d2h"] / nt},
        "timed_batches": ds["timed_batches"],
        "int_rates_tops": rates,
    }
    kernels.update(isolated_kernels(dd, off, int_peak, alu_peak))
    kernels["mandelbrot"] = mandel_measure(sm_mhz, with_cpu=not args.no_cpu_baseline)
    sha_blocks_per_byte = ds["sha1_blocks"] / max(ds["bytes"], 1)
    path_ops = value * 1e9 * (SCAN_OPS_PER_BYTE + sha_blocks_per_byte * SHA1_OPS_PER_BLOCK) / 1e12
    kernels["path"] = {"bound": "alu", "achieved": path_ops, "peak": int_peak, "unit": "Tops/s",
                       "frac": path_ops / int_peak,
                       "ops_per_byte": SCAN_OPS_PER_BYTE + sha_blocks_per_byte * SHA1_OPS_PER_BLOCK,
                       "note": "whole step: algorithmic scan + SHA-1 int ops at `value`"}
    # dominant kernel: SHA-1 (largest share of the step, profiles/); achieved =
    # its algorithmic ops per launch / launch duration of full-GPU launches
    kd = kernels["sha1"]
    traffic = None
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp):  # DRAM bytes per launch from the committed ncu capture,
        tj = json.load(open(tp))  # scaled from its batch size to this launch's bytes
        if "sha1" in tj:
            traffic = tj["sha1"] / tj["capture_batch_bytes"] * kd["launch_bytes"]
    alu_ach = kd["achieved"] * SHA1_ALU_OPS_PER_BLOCK / SHA1_OPS_PER_BLOCK
    roofline = {"kernel": "sha1_kernel", "bound": "alu", "achieved": kd["achieved"],
                "peak": int_peak, "unit": "Tops/s", "frac": kd["achieved"] / int_peak,
                "alu_pipe_view": {"achieved": alu_ach, "peak": alu_peak,
                                  "frac": alu_ach / alu_peak,
                                  "ops_per_block": SHA1_ALU_OPS_PER_BLOCK},
                "traffic": traffic,
                "peak_source": "measured (dedup_probe_int_rates, this run): SHA-1's op mix "
                               f"(432 ALU + 165 FMA ops per block) at the measured LOP3 "
                               f"{rates['lop3']:.1f}, IMAD {rates['imad']:.1f} and mixed-issue "
                               f"{rates['mix_lop3_imad']:.1f} T ops/s",
                "launch": f"{kd['launch_bytes'] / MiB:.0f} MiB of C3 chunks per launch, "
                          f"{kd['launch_us']:.0f} us per launch (CUDA events, "
                          "12 concurrent launches on their own streams)"}

    # ---- the other BASELINE.json configs ----
    cfgs = config_lines(args.steps)
    cfgs["C2_batch_sweep_gbs"] = batch_sweep(synthgen.config_stream("C2"))
    try:
        cfgs["C3_carry_over"] = carry_throughput(data)
    except Exception as e:  # report, keep the bench line
        cfgs["C3_carry_over"] = {"error": str(e)[:200]}

    # ---- end-to-end through the host-fed C ABI ----
    e2e_steps = args.e2e_steps or args.steps
    pin = d.host_empty(len(data))
    pin[:] = data
    submit_host = lambda b: d.submit_buffer(  # noqa: E731
        pin[int(off[plan[b][0]]):int(off[plan[b][1]])], subs[b][1])
    ems, de, _ = timed_passes(d, submit_host, nb, e2e_steps, args.warmup)
    e2e_value = de["bytes"] / (ems / 1e3) / 1e9
    e2e = {"value": e2e_value, "unit": "GB/s",
           "h2d_bytes_per_step": (de["bytes"] + 8 * (de["items"] + de["batches"])) / e2e_steps,
           "d2h_bytes_per_step": (33 * de["chunks"] + 4 * de["items"] + 8 * de["batches"])
           / e2e_steps,
           "steps": e2e_steps, "chunks_per_s": de["chunks"] / (ems / 1e3),
           "api": "dedup_submit_batch (pinned host buffers) + dedup_drain",
           "pcie_h2d_gbs": h2d_bandwidth(pin, dd)}
    d.close()

    line = {
        "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "chunks_per_s": chunks_per_s,
        "dup_ratio": ds["dup_chunks"] / max(ds["chunks"], 1),
        "config": {"workload": WORKLOAD_DESC, "batch_bytes": BATCH_BYTES,
                   "batch_items": BATCH_ITEMS, "slots": SLOTS, "batches_per_step": nb,
                   "parallelism": "1 GPU",
                   "l2": "inputs larger than L2 (672 MiB stream, 126 MB L2)"},
        "clocks": clocks, "gpu_launches": launches, "roofline": roofline,
        "configs": cfgs, "kernels": kernels, "e2e": e2e,
    }
    if not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(data, off)
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
