"""Multi-GPU orchestration of the dedup hot path (rows A5-A8).

Batches (whole items) are processed in WAVES: in wave w every rank r runs
its own batch through the device ops of include/dedup.h, collapses equal
digests of the batch to one representative (the smallest chunk index, i.e.
the smallest id; row A5 local combine, ``dedup_op_local_combine``), then the
representatives' digests are routed to their owner GPU,
owner(d) = floor(BE32(d[0..3]) * G / 2^32) (row A5, kernel
``dedup_op_route``), exchanged with an all-to-all (row A6),
inserted + looked up in the owner's table shard (row A7, ``dedup_op_owner``),
and the first-occurrence ids are sent back and scattered to chunk order,
every chunk taking its representative's reply (row A8, ``dedup_op_scatter``).
The combine bounds the exchange and the owner's table work by the batch's
distinct digests: an all-duplicate stream sends one record per wave instead
of every chunk to one hot owner (SURVEY 8(e) "skew").  Owners insert every record of a wave before
looking any of them up, and waves are processed in order, so the result is
the sequential stream-order answer (reading O12) whatever the GPU
count.  The paper itself has no inter-GPU step (GPUs take batches
round-robin); the exchange is needed because the
duplicate check is global (reading O11).

The per-rank work is split in three phases so that the same code runs
  * with ``TorchDistExchange``: one process per GPU, torch.distributed
    all_to_all_single (NCCL over NVLink on B200, gloo in the CPU tests), and
  * with ``LoopbackExchange``: G logical ranks on ONE GPU in one process (the
    GPU parity test of the routing).
"""
from __future__ import annotations

import ctypes
import os
import time
from dataclasses import dataclass

import numpy as np

REC_WORDS = 4  # a dedup_record is 32 bytes = 4 int64 words


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


class TorchDistExchange:
    """All-to-all of variable-size segments with torch.distributed.

    ``send`` is a 2-D tensor [n, w] whose rows are grouped by destination
    rank (``counts[r]`` rows for rank r); returns the received rows grouped
    by source rank and the per-source counts.  Counts are exchanged first
    (one small all-to-all), then the payload.
    """

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)

    def counts(self, send_counts):
        import torch
        sc = torch.as_tensor(send_counts, dtype=torch.int64)
        dev = self._device()
        sc = sc.to(dev)
        rc = torch.empty_like(sc)
        self.dist.all_to_all_single(rc, sc, group=self.group)
        return rc.cpu().tolist()

    def payload(self, send, send_counts, recv_counts):
        import torch
        recv = torch.empty((int(sum(recv_counts)),) + tuple(send.shape[1:]), dtype=send.dtype,
                           device=send.device)
        self.dist.all_to_all_single(recv, send.contiguous(),
                                    output_split_sizes=[int(x) for x in recv_counts],
                                    input_split_sizes=[int(x) for x in send_counts],
                                    group=self.group)
        return recv

    def alltoall(self, sends, counts):
        """Pipeline interface (one local rank per process): returns
        ([recv], [recv_counts])."""
        rc = self.counts(counts[0])
        return [self.payload(sends[0], counts[0], rc)], [rc]

    def _device(self):
        import torch
        backend = self.dist.get_backend(self.group)
        return torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else \
            torch.device("cpu")


def loopback_all_to_all(sends, counts):
    """In-process all-to-all for G logical ranks: sends[s] rows grouped by
    destination with counts[s][d] rows each; returns (recvs, recv_counts)."""
    import torch
    G = len(sends)
    offs = [np.concatenate([[0], np.cumsum(c)]).astype(np.int64) for c in counts]
    recvs, rcounts = [], []
    for d in range(G):
        parts = [sends[s][int(offs[s][d]):int(offs[s][d + 1])] for s in range(G)]
        recvs.append(torch.cat(parts, 0) if parts else sends[d][:0])
        rcounts.append([int(counts[s][d]) for s in range(G)])
    return recvs, rcounts


class LoopbackExchange:
    """Pipeline interface for G logical ranks in one process (one GPU)."""

    def alltoall(self, sends, counts):
        return loopback_all_to_all(sends, counts)


class RankState:
    """Device buffers + ctx of one rank (owner of one table shard)."""

    def __init__(self, dedup, batch_bytes: int, batch_items: int, device, num_owners: int,
                 combine: bool = True):
        import torch
        self.d = dedup
        self.G = num_owners
        self.combine = combine  # row A5 local combine: one record per distinct digest
        self.dev = device
        cap = batch_bytes // 32 + batch_items + 2
        self.cap = cap
        i32 = dict(dtype=torch.int32, device=device)
        i64 = dict(dtype=torch.int64, device=device)
        self.cut = torch.zeros(cap, **i32)
        self.n = torch.zeros(1, **i32)
        self.chunk_start = torch.zeros(cap, **i32)
        self.chunk_id = torch.zeros(cap, **i64)
        self.item_first = torch.zeros(batch_items + 1, **i32)
        self.digest = torch.zeros(cap * 20, dtype=torch.uint8, device=device)
        self.send = torch.zeros((cap, REC_WORDS), **i64)
        self.send_off = torch.zeros(self.G + 1, **i32)
        self.send_pos = torch.zeros(cap, **i32)
        self.rep = torch.zeros(cap, **i32) if combine else None
        self.first_id = torch.zeros(cap, **i64)
        self.is_dup = torch.zeros(cap, dtype=torch.uint8, device=device)
        self.item_off_dev = torch.zeros(batch_items + 1, **i64)

    # phase 1: rows A2-A5 on this rank's batch
    def local(self, data, item_off: np.ndarray, first_seq: int):
        import torch
        self.first_seq = first_seq
        self.item_off = np.asarray(item_off, np.uint64)
        n_items = len(self.item_off) - 1
        nbytes = int(self.item_off[-1])
        self.item_off_dev[:n_items + 1].copy_(torch.from_numpy(self.item_off.view(np.int64)))
        d = self.d
        d.op_chunk(data, nbytes, self.item_off_dev, n_items, self.cut, self.cap, self.n)
        d.op_chunk_meta(self.item_off_dev, n_items, self.cut, self.n, self.cap, first_seq,
                        self.chunk_start, self.chunk_id, self.item_first)
        d.op_sha1(data, nbytes, self.cut, self.n, self.cap, self.digest)
        if self.combine:
            d.op_local_combine(self.digest, self.n, self.cap, self.rep)
        d.op_route(self.digest, self.chunk_id, self.n, self.cap, self.G, self.send,
                   self.send_off, self.send_pos, rep=self.rep)
        off = self.send_off.cpu().numpy().astype(np.int64)   # host sync (counts)
        self.n_host = int(off[-1])  # records sent (distinct digests with combine)
        self.send_counts = np.diff(off).tolist()
        return self.send[:self.n_host], self.send_counts

    # phase 2: row A7 on the records this rank owns
    def owner(self, recv):
        import torch
        reply = torch.zeros(len(recv), dtype=torch.int64, device=self.dev)
        if len(recv):
            self.d.op_owner(recv, len(recv), reply)
        return reply

    # phase 3: row A8 + read-back of this rank's results
    def finish(self, reply_back) -> WaveOut:
        n_sent = self.n_host
        n = int(self.n.item())
        if n:
            self.d.op_scatter(reply_back, self.send_pos, self.chunk_id, self.n, self.cap,
                              self.first_id, self.is_dup, rep=self.rep)
        n_items = len(self.item_off) - 1
        self.sent_records = n_sent
        return WaveOut(
            first_seq=self.first_seq,
            item_len=np.diff(self.item_off),
            item_first=self.item_first[:n_items].cpu().numpy().view(np.uint32).copy(),
            chunk_start=self.chunk_start[:n].cpu().numpy().view(np.uint32).copy(),
            digest=self.digest[:20 * n].cpu().numpy().reshape(n, 20).copy(),
            first_id=self.first_id[:n].cpu().numpy().view(np.uint64).copy(),
            is_dup=self.is_dup[:n].cpu().numpy().copy())


def run_wave(x, state, data, item_off, first_seq: int) -> WaveOut:
    """One wave on one rank: local rows A2-A5, record all-to-all (A6), owner
    insert + lookup (A7), reply all-to-all and scatter (A8).  Every rank of
    the group must call it for the same wave."""
    send, send_counts = state.local(data, item_off, first_seq)
    recv_counts = x.counts(send_counts)
    recv = x.payload(send, send_counts, recv_counts)
    reply = state.owner(recv)
    reply_back = x.payload(reply, recv_counts, send_counts)
    return state.finish(reply_back)


class DistDedup:
    """One rank of the multi-GPU dedup (one process per GPU)."""

    def __init__(self, exchange: TorchDistExchange, device_index: int, batch_bytes: int,
                 batch_items: int, table_capacity: int, **cfg):
        import torch

        from .api import Dedup
        self.x = exchange
        self.G = exchange.world
        self.dedup = Dedup(device_index, batch_bytes=batch_bytes, batch_items=batch_items,
                           slots=1, table_capacity=table_capacity, host_fed=False,
                           owner_rank=exchange.rank, num_owners=self.G, **cfg)
        self.state = RankState(self.dedup, batch_bytes, batch_items,
                               torch.device("cuda", device_index), self.G)

    def wave(self, data, item_off, first_seq: int) -> WaveOut:
        return run_wave(self.x, self.state, data, item_off, first_seq)

    def end_stream(self):
        self.dedup.op_table_reset()

    def close(self):
        self.dedup.close()


def loopback_waves(states, batches):
    """Run one wave on G logical ranks sharing one GPU.

    states: list of RankState (rank r owns shard r); batches: list of
    (data_tensor, item_off, first_seq) per rank.  Returns a WaveOut per rank.
    """
    sends, counts = [], []
    for st, (data, off, seq) in zip(states, batches):
        s, c = st.local(data, off, seq)
        sends.append(s)
        counts.append(c)
    recvs, rcounts = loopback_all_to_all(sends, counts)
    replies = [st.owner(r) for st, r in zip(states, recvs)]
    # reverse: owner d's reply rows are grouped by source rank s
    back_counts = [[rcounts[d][s] for s in range(len(states))] for d in range(len(states))]
    backs, _ = loopback_all_to_all(replies, back_counts)
    return [st.finish(b) for st, b in zip(states, backs)]


# ---------------------------------------------------------------------------
# Pipelined waves.  run_wave() finishes a wave before the next one starts, so
# a GPU holds one batch at a time -- latency-bound (a batch's SHA-1 lasts as
# long as its longest chunk).  WavePipeline keeps `depth` waves in flight per
# local rank: the local rows A2-A5 of wave w + depth - 1 run on their own
# streams while the exchange of wave w (A6-A8) runs on the owner stream; the
# host synchronises only on wave w's route counts (to size the all-to-all)
# and on its results.  Owner work stays in wave order on one stream per rank
# (every record of wave w is inserted and looked up before wave w + 1's), so
# results are the sequential stream-order answer (reading O12).


class _Slot:
    """One in-flight wave of one local rank: a ctx of its own (the op
    workspace), a stream, RankState buffers, pinned staging and events."""

    def __init__(self, device_index, batch_bytes, batch_items, G, sha_lane_bytes, combine):
        import torch

        from .api import Dedup
        self.ctx = Dedup(device_index, batch_bytes=batch_bytes, batch_items=batch_items, slots=1,
                         table_capacity=1 << 10, host_fed=False, num_owners=G,
                         sha_lane_bytes=sha_lane_bytes)
        dev = torch.device("cuda", device_index)
        self.state = RankState(self.ctx, batch_bytes, batch_items, dev, G, combine=combine)
        self.stream = torch.cuda.Stream(device=dev)
        self.e_local = torch.cuda.Event()
        self.e_done = torch.cuda.Event()
        cap = self.state.cap
        pin = dict(pin_memory=True)
        self.h_off = torch.zeros(batch_items + 1, dtype=torch.int64, **pin)
        self.h_send_off = torch.zeros(G + 1, dtype=torch.int32, **pin)
        self.h_n = torch.zeros(1, dtype=torch.int32, **pin)
        self.h_item_first = torch.zeros(batch_items + 1, dtype=torch.int32, **pin)
        self.h_chunk_start = torch.zeros(cap, dtype=torch.int32, **pin)
        self.h_digest = torch.zeros(cap * 20, dtype=torch.uint8, **pin)
        self.h_first_id = torch.zeros(cap, dtype=torch.int64, **pin)
        self.h_is_dup = torch.zeros(cap, dtype=torch.uint8, **pin)
        self.busy = False

    def local(self, data, item_off, first_seq):
        """Rows A2-A5 on this slot's stream; no host synchronisation."""
        import torch
        st, S = self.state, self.stream
        st.first_seq = first_seq
        st.item_off = np.asarray(item_off, np.uint64)
        n_items = len(st.item_off) - 1
        nbytes = int(st.item_off[-1])
        self.h_off[:n_items + 1].copy_(torch.from_numpy(st.item_off.view(np.int64)))
        d = self.ctx
        with torch.cuda.stream(S):
            st.item_off_dev[:n_items + 1].copy_(self.h_off[:n_items + 1], non_blocking=True)
            d.op_chunk(data, nbytes, st.item_off_dev, n_items, st.cut, st.cap, st.n, stream=S)
            d.op_chunk_meta(st.item_off_dev, n_items, st.cut, st.n, st.cap, first_seq,
                            st.chunk_start, st.chunk_id, st.item_first, stream=S)
            d.op_sha1(data, nbytes, st.cut, st.n, st.cap, st.digest, stream=S)
            if st.combine:
                d.op_local_combine(st.digest, st.n, st.cap, st.rep, stream=S)
            d.op_route(st.digest, st.chunk_id, st.n, st.cap, st.G, st.send, st.send_off,
                       st.send_pos, rep=st.rep, stream=S)
            self.h_send_off.copy_(st.send_off, non_blocking=True)
            self.h_n.copy_(st.n, non_blocking=True)
            self.e_local.record(S)
        self.busy = True

    def counts(self):
        """Host: wait for this wave's route; per-owner record counts."""
        self.e_local.synchronize()
        off = self.h_send_off.numpy().astype(np.int64)
        self.state.n_host = int(off[-1])
        self.state.send_counts = np.diff(off).tolist()
        return self.state.send_counts

    def finish_async(self, reply_back, stream):
        """Row A8 + D2H of the results on the owner stream."""
        st = self.state
        n = int(self.h_n[0])
        if n:
            self.ctx.op_scatter(reply_back, st.send_pos, st.chunk_id, st.n, st.cap,
                                st.first_id, st.is_dup, rep=st.rep, stream=stream)
        n_items = len(st.item_off) - 1
        self.h_item_first[:n_items].copy_(st.item_first[:n_items], non_blocking=True)
        self.h_chunk_start[:n].copy_(st.chunk_start[:n], non_blocking=True)
        self.h_digest[:20 * n].copy_(st.digest[:20 * n], non_blocking=True)
        self.h_first_id[:n].copy_(st.first_id[:n], non_blocking=True)
        self.h_is_dup[:n].copy_(st.is_dup[:n], non_blocking=True)
        self.e_done.record(stream)
        self.n = n

    def result(self) -> WaveOut:
        self.e_done.synchronize()
        st, n = self.state, self.n
        n_items = len(st.item_off) - 1
        self.busy = False
        return WaveOut(
            first_seq=st.first_seq, item_len=np.diff(st.item_off),
            item_first=self.h_item_first[:n_items].numpy().view(np.uint32).copy(),
            chunk_start=self.h_chunk_start[:n].numpy().view(np.uint32).copy(),
            digest=self.h_digest[:20 * n].numpy().reshape(n, 20).copy(),
            first_id=self.h_first_id[:n].numpy().view(np.uint64).copy(),
            is_dup=self.h_is_dup[:n].numpy().copy())

    def close(self):
        self.ctx.close()


class WavePipeline:
    """`depth` waves in flight per local rank (rows A2-A9 at G > 1).

    owners: one Dedup ctx per LOCAL rank, owning that rank's table shard
    (owner_rank, num_owners = G); exchange: TorchDistExchange (one local rank
    per process, NCCL) or LoopbackExchange (G local ranks on one GPU).
    submit(batches) takes one (data_tensor, item_off, first_seq) per local
    rank and returns the waves completed by the call (lists of WaveOut per
    local rank, in wave order); flush() completes the rest.  Data tensors
    must stay alive until their wave is returned."""

    def __init__(self, exchange, owners, device_index: int, batch_bytes: int,
                 batch_items: int, depth: int = 4, sha_lane_bytes: int = 8192,
                 combine: bool = True):
        import torch
        self.x = exchange
        self.owners = owners
        self.G = owners[0].cfg.num_owners
        self.depth = depth
        self.slots = [[_Slot(device_index, batch_bytes, batch_items, self.G, sha_lane_bytes,
                             combine) for _ in range(depth)] for _ in owners]
        dev = torch.device("cuda", device_index)
        self.owner_streams = [torch.cuda.Stream(device=dev) for _ in owners]
        self.dev = dev
        self.next_wave = 0
        self.done_wave = 0
        # host seconds: local-phase enqueue, waits for route counts / results,
        # exchange + owner enqueue (DEDUP_PIPE_TIMES=1 prints them at close)
        self.host_s = {"local": 0.0, "wait_counts": 0.0, "exchange": 0.0, "wait_results": 0.0}

    def submit(self, batches):
        out = []
        w = self.next_wave
        if w - self.done_wave >= self.depth:
            out.append(self._complete(self.done_wave))
        t0 = time.perf_counter()
        for r, (data, item_off, first_seq) in enumerate(batches):
            self.slots[r][w % self.depth].local(data, item_off, first_seq)
        self.host_s["local"] += time.perf_counter() - t0
        self.next_wave += 1
        return out

    def flush(self):
        out = []
        while self.done_wave < self.next_wave:
            out.append(self._complete(self.done_wave))
        return out

    def end_stream(self):
        """New dedup stream: completes every wave in flight (they belong to
        the old stream), then clears the table shards.  Returns the waves
        completed by the call."""
        out = self.flush()
        for o, S in zip(self.owners, self.owner_streams):
            o.op_table_reset(stream=S)
        return out

    def _complete(self, w):
        import torch
        sl = [self.slots[r][w % self.depth] for r in range(len(self.owners))]
        t0 = time.perf_counter()
        counts = [s.counts() for s in sl]                       # host sync: route of wave w
        t1 = time.perf_counter()
        self.host_s["wait_counts"] += t1 - t0
        for s, S in zip(sl, self.owner_streams):
            S.wait_event(s.e_local)
        sends = [s.state.send[:s.state.n_host] for s in sl]
        with torch.cuda.stream(self.owner_streams[0]):
            recvs, rcounts = self.x.alltoall(sends, counts)      # row A6
        replies = []
        for r, (o, S) in enumerate(zip(self.owners, self.owner_streams)):
            S.wait_stream(self.owner_streams[0])
            reply = torch.zeros(len(recvs[r]), dtype=torch.int64, device=self.dev)
            if len(recvs[r]):
                o.op_owner(recvs[r], len(recvs[r]), reply, stream=S)   # row A7
            replies.append(reply)
        for S in self.owner_streams[1:]:
            self.owner_streams[0].wait_stream(S)
        back_counts = [[rcounts[d][s] for s in range(len(sl))] for d in range(len(sl))] \
            if len(sl) > 1 else [rcounts[0]]
        with torch.cuda.stream(self.owner_streams[0]):
            backs, _ = self.x.alltoall(replies, back_counts)     # row A8 (reply)
        res = []
        for s, b in zip(sl, backs):
            s.finish_async(b, self.owner_streams[0])
        t2 = time.perf_counter()
        self.host_s["exchange"] += t2 - t1
        for s in sl:
            # the slot's next local phase must not overwrite buffers in use
            s.stream.wait_event(s.e_done)
            res.append(s.result())
        self.host_s["wait_results"] += time.perf_counter() - t2
        self.done_wave += 1
        return res

    def close(self):
        if os.environ.get("DEDUP_PIPE_TIMES"):
            print(f"WavePipeline host seconds over {self.done_wave} waves: "
                  + ", ".join(f"{k} {v:.4f}" for k, v in self.host_s.items()), flush=True)
        for row in self.slots:
            for s in row:
                s.close()


# ---------------------------------------------------------------------------
# The same wave pipeline inside the C++ library (csrc/dist.cpp), NCCL called
# directly: this class only marshals arguments and copies results out.


def nccl_unique_id() -> bytes:
    """128-byte NCCL id; rank 0 creates it and broadcasts it to the others."""
    from . import _native as N
    buf = (ctypes.c_uint8 * 128)()
    N.check(N.lib().dedup_nccl_unique_id(buf))
    return bytes(buf)


class NativeWavePipeline:
    """One rank of the C++ wave pipeline (include/dedup.h section 4).
    submit / flush / end_stream return the completed waves as lists of one
    WaveOut (this rank's), like WavePipeline with one local rank."""

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

    def close(self):
        if self._d:
            self.N.lib().dedup_dist_destroy(self._d)
            self._d = None
