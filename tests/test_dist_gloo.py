"""Multi-rank (world_size 2) CPU tests of the digest-routing orchestration
 over torch.distributed with the gloo backend.

The device kernels cannot run on CPU, so the per-rank phases are replaced by
a test-only reference (MockState: oracle chunking + SHA-1, a dict as the
owner's table shard) with the same contract as RankState; what is under test
is the exchange plumbing (TorchDistExchange) and the wave protocol
(dist.run_wave): records reach their owner, replies come back to the right
chunk, and the 2-rank result equals the sequential oracle.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synthgen
from paper_conf_ipps_rockenbachsgmtd19_b200 import dist as D


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


def owner_of(digest_row: bytes, G: int) -> int:
    return (int.from_bytes(digest_row[:4], "big") * G) >> 32


def pack_records(digests, ids):
    """[n, 4] int64 rows laid out like dedup_record (20 B digest, pad, id)."""
    n = len(ids)
    raw = np.zeros((n, 32), np.uint8)
    raw[:, :20] = digests
    raw[:, 24:32] = np.asarray(ids, np.uint64).view(np.uint8).reshape(n, 8)
    return torch.from_numpy(raw.view(np.int64).reshape(n, 4).copy())


def unpack_records(t):
    raw = t.numpy().view(np.uint8).reshape(-1, 32)
    return raw[:, :20], raw[:, 24:32].copy().view(np.uint64).reshape(-1)


# ------------------------------------------------------- exchange only -----
def _exchange_case(rank, world):
    x = D.TorchDistExchange()
    rng_of = lambda r: np.random.default_rng(1000 + r)  # noqa: E731

    def records(r):
        rng = rng_of(r)
        n = 300 + 37 * r
        dg = rng.integers(0, 256, (n, 20), dtype=np.uint8)
        ids = (np.arange(n, dtype=np.uint64) << np.uint64(8)) | np.uint64(r)
        own = np.array([owner_of(bytes(d), world) for d in dg])
        order = np.argsort(own, kind="stable")
        counts = np.bincount(own, minlength=world).tolist()
        return dg[order], ids[order], counts

    dg, ids, counts = records(rank)
    send = pack_records(dg, ids)
    rc = x.counts(counts)
    recv = x.payload(send, counts, rc)
    rdg, rids = unpack_records(recv)
    # expected: the rows of every source s destined to me, in source order
    exp_ids = []
    for s in range(world):
        sdg, sids, sc = records(s)
        off = np.concatenate([[0], np.cumsum(sc)])
        exp_ids.append(sids[off[rank]:off[rank + 1]])
    exp_ids = np.concatenate(exp_ids)
    assert np.array_equal(rids, exp_ids)
    assert all(owner_of(bytes(d), world) == rank for d in rdg)
    # replies travel back to the sender, aligned with its send order
    reply = torch.from_numpy((rids * np.uint64(7)).view(np.int64).copy())
    back = x.payload(reply, rc, counts)
    assert np.array_equal(back.numpy().view(np.uint64), ids * np.uint64(7))
    return True


def test_exchange_records_and_replies_gloo():
    out = _run("_exchange_case")
    assert all(out.values())


# ------------------------------------------- full protocol vs the oracle -----
class MockState:
    """Test-only stand-in for dist.RankState (same phase contract)."""

    def __init__(self, rank, G):
        self.rank, self.G = rank, G
        self.table = {}

    def local(self, data, item_off, first_seq):
        self.first_seq = first_seq
        self.item_off = np.asarray(item_off, np.uint64)
        starts, digs, ids, firsts = [], [], [], []
        k = 0
        for it in range(len(self.item_off) - 1):
            a, b = int(self.item_off[it]), int(self.item_off[it + 1])
            cs = oracle.chunk_item(data[a:b]) if b > a else np.zeros(0, np.uint32)
            firsts.append(k if len(cs) else 0xFFFFFFFF)
            ends = list(map(int, cs[1:])) + [b - a]
            for j, (s, e) in enumerate(zip(map(int, cs), ends)):
                starts.append(s)
                digs.append(np.frombuffer(oracle.sha1(data[a + s:a + e]), np.uint8))
                ids.append(((first_seq + it) << 32) | j)
                k += 1
        self.starts = np.array(starts, np.uint32)
        self.digs = np.array(digs, np.uint8).reshape(-1, 20)
        self.ids = np.array(ids, np.uint64)
        self.firsts = np.array(firsts, np.uint32)
        own = np.array([owner_of(bytes(d), self.G) for d in self.digs], np.int64)
        order = np.argsort(own, kind="stable")
        self.send_pos = np.empty(len(order), np.int64)
        self.send_pos[order] = np.arange(len(order))
        counts = np.bincount(own, minlength=self.G).tolist() if len(own) else [0] * self.G
        return pack_records(self.digs[order], self.ids[order]), counts

    def owner(self, recv):
        dg, ids = unpack_records(recv)
        keys = [bytes(d) for d in dg]
        for kk, i in zip(keys, ids):          # insert the whole wave first
            self.table[kk] = min(self.table.get(kk, 1 << 64), int(i))
        return torch.tensor([self.table[kk] for kk in keys], dtype=torch.uint64).view(
            torch.int64)

    def finish(self, reply_back):
        fid = reply_back.numpy().view(np.uint64)[self.send_pos]
        return D.WaveOut(self.first_seq, np.diff(self.item_off), self.firsts, self.starts,
                         self.digs, fid, (fid != self.ids).astype(np.uint8))


def _protocol_case(rank, world):
    data = synthgen.make_stream(3 << 19, seed=12, dup_frac=0.6, segment=32 * 1024)
    off = synthgen.split_items(data, 64 * 1024)
    n_items = len(off) - 1
    per_batch = 3
    batches = [(k, min(k + per_batch, n_items)) for k in range(0, n_items, per_batch)]
    x = D.TorchDistExchange()
    st = MockState(rank, world)
    out = []
    for w in range(0, len(batches), world):  # wave w: batch w + r on rank r
        b = w + rank
        if b < len(batches):
            k, j = batches[b]
            sub = data[int(off[k]):int(off[j])]
            res = D.run_wave(x, st, sub, off[k:j + 1] - off[k], k)
        else:  # idle rank still takes part in the collectives
            res = D.run_wave(x, st, np.zeros(0, np.uint8), np.zeros(1, np.uint64), n_items)
        out.extend((seq, cs, dg, dup, fid) for seq, cs, dg, dup, fid in res.items())
    return out


def test_two_rank_protocol_matches_oracle_gloo():
    out = _run("_protocol_case")
    got = sorted(out[0] + out[1], key=lambda r: r[0])
    data = synthgen.make_stream(3 << 19, seed=12, dup_frac=0.6, segment=32 * 1024)
    off = synthgen.split_items(data, 64 * 1024)
    want, counts = oracle.dedup_items([data[int(off[k]):int(off[k + 1])]
                                       for k in range(len(off) - 1)])
    assert counts["dup_chunks"] > 0
    assert [g[0] for g in got] == [w.seq for w in want]
    for (seq, cs, dg, dup, fid), w in zip(got, want):
        assert np.array_equal(cs, w.chunk_start), seq
        assert np.array_equal(dg, w.digest), seq
        assert np.array_equal(dup, w.is_dup), seq
        assert np.array_equal(fid, w.first_id), seq
