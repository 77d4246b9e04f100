"""GPU parity at the BASELINE.json sizes, in the bench's launch configuration
(64 MiB batches of 1 MiB items, device-resident), on outputs the CPU can
check one by one: every chunk's SHA-1 recomputed with hashlib, every dup
flag and first-occurrence id recomputed with a dict in stream order, the
partition invariants of every item, and the oracle's chunking of sampled
items; closed forms for the degenerate streams.

  C3  672 MiB native-sized stream (dup 0.52)
  C4  its per-GPU share on 8 GPUs: the first 2 GiB of the 16 GiB stream
  C5a 672 MiB all-unique
  C5b 672 MiB all-duplicate (every item = item 0)
  C5c(i) 672 MiB all-zero (22 M identical 32-byte chunks)
"""
import hashlib

import numpy as np
import pytest

import oracle
import synthgen
from tests import gpu_util as U

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

MiB = 1 << 20
BATCH = 64 * MiB


def run_engine(data, off):
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    with Dedup(0, batch_bytes=BATCH, batch_items=64, slots=8,
               table_capacity=max(1 << 16, len(data) // 2048)) as d:
        return U.run_device(d, torch.from_numpy(data).cuda(), off, BATCH, 64)


def verify(data, off, got, n_sample=8, seed=0):
    n_items = len(off) - 1
    assert [g.seq for g in got] == list(range(n_items))
    first = {}
    rng = np.random.default_rng(seed)
    sample = set(rng.choice(n_items, min(n_sample, n_items), replace=False).tolist())
    sample |= {0, n_items - 1}
    for k, g in enumerate(got):
        a, b = int(off[k]), int(off[k + 1])
        item = data[a:b]
        cs = g.chunk_start.astype(np.int64)
        ends = np.append(cs[1:], b - a)
        assert cs[0] == 0 and np.all(np.diff(cs) >= 32), k        # partition, min size
        if k in sample:
            assert np.array_equal(g.chunk_start, oracle.chunk_item(item)), k
        mv = memoryview(item)
        for j, (s, e) in enumerate(zip(cs, ends)):
            dg = hashlib.sha1(mv[s:e]).digest()
            assert g.digest[j].tobytes() == dg, (k, j)
            fid = first.setdefault(dg, (k << 32) | j)
            assert int(g.first_id[j]) == fid, (k, j)
            assert int(g.is_dup[j]) == (fid != ((k << 32) | j)), (k, j)


@pytest.mark.parametrize("name,nbytes", [("C3", None), ("C5a", None), ("C4", 2 << 30)])
def test_fullsize_stream(name, nbytes):
    data = synthgen.config_stream(name, nbytes=nbytes)
    off = synthgen.split_items(data)
    got = run_engine(data, off)
    verify(data, off, got)


def test_fullsize_all_duplicate():
    item0 = synthgen.make_stream(MiB, seed=52)
    data = np.tile(item0, 672)
    off = synthgen.split_items(data)
    got = run_engine(data, off)
    (w0,), _ = oracle.dedup_items([item0])
    for k, g in enumerate(got):
        assert np.array_equal(g.chunk_start, w0.chunk_start), k
        assert np.array_equal(g.digest, w0.digest), k
        if k == 0:
            assert np.array_equal(g.first_id, w0.first_id)
            assert np.array_equal(g.is_dup, w0.is_dup)
        else:    # every chunk repeats a chunk of item 0
            assert np.array_equal(g.first_id, w0.first_id), k
            assert g.is_dup.all(), k
    verify(item0, np.array([0, MiB], np.uint64), got[:1])


def test_fullsize_all_zero():
    data = np.zeros(672 * MiB, np.uint8)
    off = synthgen.split_items(data)
    got = run_engine(data, off)
    d0 = np.frombuffer(hashlib.sha1(bytes(32)).digest(), np.uint8)
    starts = np.arange(0, MiB, 32, dtype=np.uint32)
    for k, g in enumerate(got):
        assert np.array_equal(g.chunk_start, starts), k
        assert (g.digest == d0).all(), k
        assert (g.first_id == 0).all(), k
        want_dup = np.ones(len(starts), np.uint8)
        if k == 0:
            want_dup[0] = 0
        assert np.array_equal(g.is_dup, want_dup), k
