"""GPU parity at the BASELINE.json sizes, in the launch configuration bench.py
times (64 MiB batches of 1 MiB items, device-resident, bench.engine_kwargs),
compared ELEMENT BY ELEMENT with the oracle on every item: chunk starts,
digests, dup flags and first-occurrence ids.  The oracle runs its threaded
driver (chunking + SHA-1 of the items on all host cores, the dedup table
sequential in stream order, pinned to the sequential
oracle in tests/test_oracle_pins.py).

  C3     672 MiB native-sized stream (dup 0.52)          -- the bench headline
  C4     its per-GPU share on 8 GPUs: the first 2 GiB of the 16 GiB stream
  C5a    672 MiB all-unique
  C5b    672 MiB all-duplicate (every item = item 0)      (+ closed form)
  C5c(i) 672 MiB all-zero (22 M identical 32-byte chunks) (+ closed form)
"""
import hashlib

import numpy as np
import pytest

import bench
import oracle
import synthgen
from tests import gpu_util as U

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

MiB = 1 << 20


def run_engine(data, off):
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    with Dedup(0, **bench.engine_kwargs(len(data))) as d:
        return U.run_device(d, torch.from_numpy(data).cuda(), off, bench.BATCH_BYTES,
                            bench.BATCH_ITEMS)


def compare_with_oracle(data, off, got):
    """Every output of every item against the oracle run on the same bytes."""
    n_items = len(off) - 1
    assert [g.seq for g in got] == list(range(n_items))
    s = oracle.Stream()
    want = s.items_parallel(0, data, off)
    s.close()
    assert sum(g.n_chunks for g in got) == len(want.chunk_start)
    for k, g in enumerate(got):
        assert g.item_len == int(off[k + 1] - off[k]), k
        cs, dg, dup, fid = want.item(k)
        assert np.array_equal(g.chunk_start, cs), f"chunk_start item {k}"
        assert np.array_equal(g.digest, dg), f"digest item {k}"
        assert np.array_equal(g.is_dup, dup), f"is_dup item {k}"
        assert np.array_equal(g.first_id, fid), f"first_id item {k}"
    return want


@pytest.mark.parametrize("name,nbytes", [("C3", None), ("C5a", None), ("C4", 2 << 30)])
def test_fullsize_stream(name, nbytes):
    data = synthgen.config_stream(name, nbytes=nbytes)
    off = synthgen.split_items(data)
    got = run_engine(data, off)
    want = compare_with_oracle(data, off, got)
    if name == "C5a":
        assert want.is_dup.sum() == 0          # all-unique: no duplicate chunk at all


def test_fullsize_all_duplicate():
    item0 = synthgen.make_stream(MiB, seed=52)
    data = np.tile(item0, 672)
    off = synthgen.split_items(data)
    got = run_engine(data, off)
    compare_with_oracle(data, off, got)
    (w0,), _ = oracle.dedup_items([item0])
    for k, g in enumerate(got[1:], 1):         # closed form: every chunk repeats item 0's
        assert np.array_equal(g.first_id, w0.first_id), k
        assert g.is_dup.all(), k


def test_fullsize_all_zero():
    data = np.zeros(672 * MiB, np.uint8)
    off = synthgen.split_items(data)
    got = run_engine(data, off)
    compare_with_oracle(data, off, got)
    d0 = np.frombuffer(hashlib.sha1(bytes(32)).digest(), np.uint8)
    starts = np.arange(0, MiB, 32, dtype=np.uint32)
    for k, g in enumerate(got):                # closed form: 32-byte chunks, one digest
        assert np.array_equal(g.chunk_start, starts), k
        assert (g.digest == d0).all(), k
        assert (g.first_id == 0).all(), k
        assert g.is_dup.sum() == len(starts) - (k == 0), k


def test_fullsize_op_chunk_one_launch():
    """The whole 672 MiB C3 stream chunked by ONE op_chunk launch: the roll
    kernel's many-tasks-per-warp configuration (512-byte lanes; the engine's
    64 MiB batches use 2 KiB lanes), every cut position against the oracle."""
    from paper_conf_ipps_rockenbachsgmtd19_b200 import Dedup
    data = synthgen.config_stream("C3")
    off = synthgen.split_items(data)
    nbytes, n_items = len(data), len(off) - 1
    with Dedup(0, batch_bytes=nbytes, batch_items=n_items + 1, slots=1, table_capacity=1 << 12,
               host_fed=False) as d:
        dev = torch.from_numpy(data).cuda()
        offt = torch.from_numpy(off.astype(np.int64)).cuda()
        cap = nbytes // 32 + n_items + 2
        cut = torch.zeros(cap, dtype=torch.int32, device="cuda")
        n = torch.zeros(1, dtype=torch.int32, device="cuda")
        d.op_chunk(dev, nbytes, offt, n_items, cut, cap, n)
        torch.cuda.synchronize()
        got = cut[:int(n.item())].cpu().numpy().astype(np.int64)
    s = oracle.Stream()
    want = s.items_parallel(0, data, off)
    s.close()
    exp = np.concatenate([int(off[k]) + want.item(k)[0].astype(np.int64) for k in range(n_items)])
    assert np.array_equal(got, exp)
