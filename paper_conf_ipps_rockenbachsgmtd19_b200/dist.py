"""Multi-GPU orchestration of the dedup hot path (rows A5-A8).

The protocol lives in the C++ engine (csrc/mg.cpp): in wave w every rank
runs its own batch through the local rows (chunking, SHA-1, local combine of
equal digests, route by owner = floor(BE32(d[0..3]) G / 2^32)), the records
go to their owner ranks (A6), each owner inserts then looks up every record
of the wave in its table shard (A7), and the first-occurrence ids come back
and are scattered to chunk order (A8).  Two front ends:
  * one process, G ranks: ``Dedup(num_devices=G, ...)`` (include/dedup.h
    dedup_init), results merged in seq order by dedup_drain;
  * one process per GPU under torchrun: ``NativeWavePipeline`` below
    (dedup_dist_*), NCCL between the processes.
The paper itself has no inter-GPU step (GPUs take batches round-robin,
PAPER.md P:185); the exchange is needed because the duplicate check is
global (reading O11).
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass

import numpy as np



@dataclass
class WaveOut:
    """Per-rank output of one wave (host numpy arrays, chunk order)."""
    first_seq: int
    item_len: np.ndarray      # u64 [n_items]
    item_first: np.ndarray    # u32 [n_items] (0xFFFFFFFF = empty item)
    chunk_start: np.ndarray   # u32 [n]
    digest: np.ndarray        # u8 [n, 20]
    first_id: np.ndarray      # u64 [n]
    is_dup: np.ndarray        # u8 [n]

    def items(self):
        """Per-item (seq, chunk_start, digest, is_dup, first_id) tuples."""
        n = len(self.chunk_start)
        nxt = n
        bounds = [None] * len(self.item_len)
        for k in range(len(self.item_len) - 1, -1, -1):
            f = int(self.item_first[k])
            if f == 0xFFFFFFFF:
                bounds[k] = (nxt, nxt)
            else:
                bounds[k] = (f, nxt)
                nxt = f
        for k, (a, b) in enumerate(bounds):
            yield (self.first_seq + k, self.chunk_start[a:b], self.digest[a:b],
                   self.is_dup[a:b], self.first_id[a:b])


# ---------------------------------------------------------------------------
# The wave pipeline of the C++ multi-GPU engine (csrc/mg.cpp), one process per
# GPU, NCCL called directly: this class only marshals arguments and copies
# results out.


def nccl_unique_id() -> bytes:
    """128-byte NCCL id; rank 0 creates it and broadcasts it to the others."""
    from . import _native as N
    buf = (ctypes.c_uint8 * 128)()
    N.check(N.lib().dedup_nccl_unique_id(buf))
    return bytes(buf)


class NativeWavePipeline:
    """One rank of the C++ wave pipeline (include/dedup.h section 4).
    submit / flush / end_stream return the completed waves as lists of one
    WaveOut (this rank's)."""

    def __init__(self, nccl_id: bytes, nranks: int, rank: int, device_index: int,
                 batch_bytes: int, batch_items: int, table_capacity: int, depth: int = 4,
                 **cfg):
        from . import _native as N
        self.N = N
        c = N.Config()
        N.lib().dedup_config_default(ctypes.byref(c))
        for k, v in dict(device=device_index, slots=1, batch_bytes=1 << 20, batch_items=1,
                         table_capacity=table_capacity, host_fed=0, owner_rank=rank,
                         num_owners=nranks, **cfg).items():
            setattr(c, k, v)
        idb = (ctypes.c_uint8 * 128).from_buffer_copy(nccl_id)
        self._d = ctypes.c_void_p()
        st = N.lib().dedup_dist_create(ctypes.byref(c), idb, nranks, rank, depth, batch_bytes,
                                       batch_items, ctypes.byref(self._d))
        if st != N.DEDUP_OK:
            raise N.DedupError(st, "dedup_dist_create failed")
        self._keep = []

    def _check(self, st):
        if st != self.N.DEDUP_OK:
            raise self.N.DedupError(st, self.N.lib().dedup_dist_last_error(self._d).decode())

    def _result(self):
        N = self.N
        r = N.WaveResult()
        self._check(N.lib().dedup_dist_result(self._d, ctypes.byref(r)))
        n, ni = r.n_chunks, r.n_items
        arr = lambda p, k, dt: np.ctypeslib.as_array(p, shape=(k,)).astype(dt, copy=True) \
            if k else np.zeros(0, dt)  # noqa: E731
        off = arr(r.item_off, ni + 1, np.uint64)
        return [WaveOut(first_seq=r.first_seq, item_len=np.diff(off),
                        item_first=arr(r.item_first_chunk, ni, np.uint32),
                        chunk_start=arr(r.chunk_start, n, np.uint32),
                        digest=arr(r.digest, 20 * n, np.uint8).reshape(n, 20),
                        first_id=arr(r.first_id, n, np.uint64),
                        is_dup=arr(r.is_dup, n, np.uint8))]

    def _counts(self):
        N = self.N
        ni, nc, nb = ctypes.c_uint32(), ctypes.c_uint32(), ctypes.c_uint64()
        self._check(N.lib().dedup_dist_last_counts(self._d, ctypes.byref(ni), ctypes.byref(nc),
                                                   ctypes.byref(nb)))
        return nb.value, nc.value

    def submit(self, batches, collect: bool = True):
        """collect=False: completed waves are returned as (bytes, chunks)
        without waiting for their results to reach host memory."""
        (data, item_off, first_seq), = batches
        import torch
        off = np.ascontiguousarray(item_off, np.uint64)
        done = ctypes.c_uint32()
        prod = torch.cuda.current_stream().cuda_stream
        self._check(self.N.lib().dedup_dist_submit(
            self._d, data.data_ptr() if data.numel() else 0, int(off[-1]), off.ctypes.data,
            len(off) - 1, first_seq, prod, ctypes.byref(done)))
        self._keep.append((data, off))
        self._keep = self._keep[-64:]
        if not done.value:
            return []
        return [self._result()] if collect else [self._counts()]

    def flush(self, collect: bool = True):
        out = []
        while True:
            done = ctypes.c_uint32()
            self._check(self.N.lib().dedup_dist_flush(self._d, ctypes.byref(done)))
            if not done.value:
                return out
            out.append(self._result() if collect else self._counts())

    def end_stream(self, collect: bool = True, drain: bool = True):
        """New dedup stream.  drain=False keeps the waves in flight (their
        results come out of later submit/flush calls); the table reset is
        then issued in wave order before the next stream's first wave."""
        out = self.flush(collect) if drain else []
        self._check(self.N.lib().dedup_dist_end_stream(self._d))
        return out

    def join(self, stream=None):
        """Make `stream` (default: torch's current stream) wait for the
        results of every completed wave (dedup_dist_join)."""
        import torch
        s = stream if stream is not None else torch.cuda.current_stream().cuda_stream
        self._check(self.N.lib().dedup_dist_join(self._d, s))

    def kernel_launches(self) -> int:
        return int(self.N.lib().dedup_dist_kernel_launches(self._d))

    def a2a_bytes(self) -> int:
        """Record + reply bytes this rank sent to other ranks so far."""
        return int(self.N.lib().dedup_dist_a2a_bytes(self._d))

    def close(self):
        if self._d:
            self.N.lib().dedup_dist_destroy(self._d)
            self._d = None
