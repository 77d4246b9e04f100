"""Row NEXT-2, carry-over chunking: the whole byte stream is
ONE chunking domain and the caller may cut it into pieces anywhere.

The item model of the engine (reading O8: an item is the paper's fixed
1 MB batch, its start a forced cut) makes results independent of how whole
items are grouped into GPU batches; this mode removes the item boundaries
instead (PARSEC's serial pipeline carries the unfinished tail from one
buffer to the next [EXT]; the paper changed that fragmentation).
With min chunk = window = 32 the chunker's state at a cut is exactly the
state at an item start (the hash restarts and the next 32 positions are
blocked), so every piece is chunked as one item that starts at the last
cut of the previous piece: the bytes after that cut are carried over and
re-chunked together with the next piece, and only chunks that end at a cut
are reported.  Every step runs in the library's kernels through the op API
(dedup_op_chunk / _chunk_meta / _sha1 / _table_insert_lookup); this class
is host orchestration (which bytes go in the next call) and marshalling.

Chunk ids are (piece << 32) | index-in-piece, so their order is the stream
order and the table's minimum id is the first occurrence (reading O12);
results report first occurrences as global chunk indices.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass
class StreamChunks:
    offset: np.ndarray      # u64 [n] stream offset of each completed chunk
    length: np.ndarray      # u64 [n]
    digest: np.ndarray      # u8 [n, 20]
    is_dup: np.ndarray      # u8 [n]
    first_index: np.ndarray  # u64 [n] global index of the first chunk with this digest


class CarryChunker:
    """Feed a device byte stream in arbitrary pieces; get the chunks of the
    whole stream (identical for any cut of the stream into pieces)."""

    def __init__(self, device: int = 0, max_piece: int = 64 << 20,
                 table_capacity: int = 1 << 20):
        import torch

        from .api import Dedup
        # a piece plus the carried tail must fit one batch; the tail is at
        # most one (unfinished) chunk, unbounded without max_chunk
        self.cap_bytes = 2 * max_piece
        self.d = Dedup(device, batch_bytes=self.cap_bytes, batch_items=2, slots=1,
                       table_capacity=table_capacity, host_fed=False, sha_lane_bytes=8192)
        self.dev = torch.device("cuda", device)
        cap = self.cap_bytes // 32 + 4
        self.cap = cap
        i32 = dict(dtype=torch.int32, device=self.dev)
        self.cut = torch.zeros(cap, **i32)
        self.n = torch.zeros(1, **i32)
        self.nf = torch.zeros(1, **i32)
        self.chunk_start = torch.zeros(cap, **i32)
        self.chunk_id = torch.zeros(cap, dtype=torch.int64, device=self.dev)
        self.item_first = torch.zeros(2, **i32)
        self.digest = torch.zeros(cap * 20, dtype=torch.uint8, device=self.dev)
        self.first_id = torch.zeros(cap, dtype=torch.int64, device=self.dev)
        self.is_dup = torch.zeros(cap, dtype=torch.uint8, device=self.dev)
        self.item_off = torch.zeros(2, dtype=torch.int64, device=self.dev)
        self.buf = torch.zeros(self.cap_bytes + 16, dtype=torch.uint8, device=self.dev)
        self.carry = 0          # bytes of the unfinished chunk at buf[0:carry]
        self.base = 0           # stream offset of buf[0]
        self.piece = 0          # pieces fed (the id's high word)
        self.index_base = []    # (piece, global index of its first chunk)
        self.n_chunks = 0

    def feed(self, data, final: bool = False) -> StreamChunks:
        """data: a CUDA uint8 tensor (may be empty).  Returns the chunks that
        are complete after this piece (all remaining ones if final)."""
        import torch
        k = int(data.numel())
        nb = self.carry + k
        if nb > self.cap_bytes:
            raise ValueError(f"piece + carried tail ({nb} B) exceeds {self.cap_bytes} B")
        if k:
            self.buf[self.carry:nb].copy_(data)
        if nb == 0:
            return self._empty()
        d, cap = self.d, self.cap
        self.item_off.copy_(torch.tensor([0, nb], dtype=torch.int64))
        d.op_chunk(self.buf, nb, self.item_off, 1, self.cut, cap, self.n)
        n = int(self.n.item())
        if final:
            nf, end = n, nb
        else:
            nf = n - 1                                   # the last chunk may continue
            end = int(self.cut[n - 1].item())             # its start: the carry point
        if nf == 0:                                      # no completed chunk yet
            self._carry_from(0, nb)
            return self._empty()
        self.nf.fill_(nf)
        d.op_chunk_meta(self.item_off, 1, self.cut, self.nf, cap, self.piece, self.chunk_start,
                        self.chunk_id, self.item_first)
        d.op_sha1(self.buf, end, self.cut, self.nf, cap, self.digest)
        d.op_table(self.digest, self.chunk_id, self.nf, cap, self.first_id, self.is_dup)
        starts = self.cut[:nf].cpu().numpy().astype(np.uint64)
        ends = np.append(starts[1:], np.uint64(end))
        fid = self.first_id[:nf].cpu().numpy().view(np.uint64)
        out = StreamChunks(
            offset=starts + np.uint64(self.base), length=ends - starts,
            digest=self.digest[:20 * nf].cpu().numpy().reshape(nf, 20).copy(),
            is_dup=self.is_dup[:nf].cpu().numpy().copy(),
            first_index=self._global_index(fid, nf))
        self.n_chunks += nf
        self.piece += 1
        if final:
            self.carry, self.base = 0, self.base + nb
        else:
            self._carry_from(end, nb)
        return out

    def _global_index(self, fid, nf):
        self.index_base.append((self.piece, self.n_chunks))
        pieces = np.array([p for p, _ in self.index_base], np.uint64)
        bases = np.array([b for _, b in self.index_base], np.uint64)
        hi = fid >> np.uint64(32)
        lo = fid & np.uint64(0xFFFFFFFF)
        return bases[np.searchsorted(pieces, hi)] + lo

    def _carry_from(self, start, nb):
        """Keep buf[start:nb] as the head of the next piece."""
        if start:
            self.buf[:nb - start].copy_(self.buf[start:nb].clone())
        self.base += start
        self.carry = nb - start

    def _empty(self):
        z = np.zeros(0, np.uint64)
        return StreamChunks(z, z.copy(), np.zeros((0, 20), np.uint8), np.zeros(0, np.uint8),
                            z.copy())

    def close(self):
        self.d.close()
